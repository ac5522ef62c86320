# setmaxnreg experiment: producers 40 regs (8 warps), consumers 72 regs, batch 8/12/16
TAG=${1:-r20d}
O=gpurun_out
run() {
  env $E timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>$O/${TAG}_err.txt | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$V $E', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt || (echo "$V $E FAILED" >> $O/${TAG}_sweep.txt; tail -3 $O/${TAG}_err.txt >> $O/${TAG}_sweep.txt)
}
V=base; E=""; run; E="TC_PROD_DIV=4"; run
for B in 8 12 16; do
  V="maxnreg40/72 B=$B"
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_MAXNREG=1 -DTC_MAXNREG_PROD=40 -DTC_MAXNREG_CONS=72 -DTC_BATCH_LONG=$B" > $O/${TAG}_make_$B.txt 2>&1
  E=""; run
done
echo done > $O/${TAG}_done.txt
