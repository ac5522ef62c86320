# A/B of 32-key steps in flight per warp in the short-class support walk (TC_UNROLL_SUP_SHORT)
TAG=${1:-r25s}
O=gpurun_out
for F in 5 3 8 5 3 8; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_UNROLL_SUP_SHORT=$F" > /dev/null 2>&1 || echo "build failed $F" >> $O/${TAG}_ab.txt
  for C in C3 C2 C5; do
  timeout 600 python bench.py --mode support --config $C --no-sharded --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C UNROLL_SUP_SHORT=$F', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
  done
done
echo done > $O/${TAG}_done.txt
