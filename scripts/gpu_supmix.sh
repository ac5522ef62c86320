# A/B of the mixed bitmap/hash batch path in the long-class support walk (TC_SUP_MIX), then the
# support parity tests with it on
TAG=${1:-r24m}
O=gpurun_out
for F in 0 1 0 1; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_SUP_MIX=$F" > /dev/null 2>&1 || echo "build failed $F" >> $O/${TAG}_ab.txt
  for C in C3 C2 C5; do
  timeout 600 python bench.py --mode support --config $C --no-sharded --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C SUP_MIX=$F', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
  done
done
timeout 900 python -m pytest tests/test_gpu_support.py -q -x > $O/${TAG}_pytest_support.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_support.txt
echo done > $O/${TAG}_done.txt
