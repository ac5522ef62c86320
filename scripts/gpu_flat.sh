# flat (short-class) kernel shape: block x CTAs/SM x unroll
TAG=${1:-r20f}
O=gpurun_out
run() {
  timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 10 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$V $C', round(d['ms_per_step'],4), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt
}
for cfg in "512 3 4" "512 3 8" "256 6 4" "256 6 8" "1024 2 4" "384 4 4"; do
  set -- $cfg
  V="block=$1 ctas=$2 unroll=$3"
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_FLAT_BLOCK=$1 -DTC_FLAT_CTAS=$2 -DTC_UNROLL_SHORT=$3" > $O/${TAG}_make.txt 2>&1
  for C in C2 C5 C3; do run; done
done
echo done > $O/${TAG}_done.txt
