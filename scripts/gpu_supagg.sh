# A/B of the (u,v) run aggregation in the long-class support walk (TC_SUP_AGG), then the support
# parity tests with it on
TAG=${1:-r23s}
O=gpurun_out
for A in 0 1 0 1; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_SUP_AGG=$A" > /dev/null 2>&1
  timeout 600 python bench.py --mode support --no-sharded --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('AGG=$A', round(d['ms_per_step'],2), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
done
timeout 900 python -m pytest tests/test_gpu_support.py -q -x > $O/${TAG}_pytest_support.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_support.txt
echo done > $O/${TAG}_done.txt
