# A/B of the all-bitmap fast path in the long-class support walk (TC_SUP_FAST), then the support
# parity tests with it on
TAG=${1:-r23t}
O=gpurun_out
for F in "-DTC_SUP_FAST=0" "-DTC_SUP_FAST=1" "-DTC_SUP_FAST=1 -DTC_UNROLL_SUP=4" "-DTC_SUP_FAST=0" "-DTC_SUP_FAST=1" "-DTC_SUP_FAST=1 -DTC_UNROLL_SUP=4" "-DTC_SUP_FAST=1"; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="$F" > /dev/null 2>&1
  timeout 600 python bench.py --mode support --no-sharded --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$F', round(d['ms_per_step'],2), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
done
timeout 900 python -m pytest tests/test_gpu_support.py -q -x > $O/${TAG}_pytest_support.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_support.txt
echo done > $O/${TAG}_done.txt
