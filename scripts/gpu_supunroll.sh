# A/B of tiles in flight per warp in the support walk with the fast path on (TC_UNROLL_SUP)
TAG=${1:-r24u}
O=gpurun_out
for F in 6 5 8 6 5 8; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_UNROLL_SUP=$F" > /dev/null 2>&1
  for C in C3 C2; do
  timeout 600 python bench.py --mode support --config $C --no-sharded --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C UNROLL_SUP=$F', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
  done
done
echo done > $O/${TAG}_done.txt
