TAG=${1:-r20k}
O=gpurun_out
for U in 4 6 8; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_UNROLL_SUP=$U" > /dev/null 2>&1
  timeout 600 python bench.py --mode support --no-sharded --no-cpu-baseline --steps 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('U=$U', round(d['ms_per_step'],2), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
done
echo done > $O/${TAG}_done.txt
