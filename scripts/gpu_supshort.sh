# A/B of the per-segment (u,v) aggregation in the short-class support walk (TC_SUP_SHORT_AGG) at C3
# and C2, the support parity tests with it on, support bench lines and one ncu capture of k_support
TAG=${1:-r23u}
O=gpurun_out
for F in 0 1 0 1; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_SUP_SHORT_AGG=$F" > /dev/null 2>&1
  for C in C3 C2; do
  timeout 600 python bench.py --mode support --config $C --no-sharded --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C SHORT_AGG=$F', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
  done
done
timeout 900 python -m pytest tests/test_gpu_support.py -q -x > $O/${TAG}_pytest_support.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_support.txt
timeout 600 python bench.py --mode support --no-sharded --out $O/${TAG}_bench_support_c3.json > /dev/null 2>&1
timeout 600 python bench.py --mode support --config C2 --no-sharded --out $O/${TAG}_bench_support_c2.json > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_support" -s 1 -c 1 -o $O/${TAG}_prof_sup_c3 python bench.py --mode support --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded > $O/${TAG}_ncu_log.txt 2>&1
echo done > $O/${TAG}_done.txt
