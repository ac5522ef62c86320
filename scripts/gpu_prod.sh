# producer-side A/B: insert unroll (row loads in flight) and staging batch
TAG=${1:-r20e}
O=gpurun_out
run() {
  env $E timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$V $C $E', round(d['ms_per_step'],4), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt
}
V=ins4; for C in C3 C2; do E=""; run; E="TC_PROD_DIV=6"; run; done
for U in 8 2; do
  V=ins$U
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_INS_UNROLL=$U" > $O/${TAG}_make_$U.txt 2>&1
  for C in C3 C2; do E=""; run; E="TC_PROD_DIV=6"; run; done
done
echo done > $O/${TAG}_done.txt
