# batch size (rebuild with -DTC_BATCH_LONG) x producer share, C3 count ms
TAG=${1:-r19j}
O=gpurun_out
run() {
  env "$@" timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$B $*', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt
}
B=8; run TC_PROD_DIV=5; run TC_PROD_DIV=4
for B in 12 16; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_BATCH_LONG=$B" > $O/${TAG}_make_$B.txt 2>&1
  grep -A1 "Function properties for .*k_countENS" build/tc_count.ptxas.txt >> $O/${TAG}_make_$B.txt
  run TC_PROD_DIV=5; run TC_PROD_DIV=4; run TC_PROD_DIV=6
done
echo done > $O/${TAG}_done.txt
