TAG=${1:-r20i}
O=gpurun_out
run() {
  env $E timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 10 "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C $E $*', round(d['ms_per_step'],4), d['parity_vs_oracle'], d['config']['keys_total']/d['config']['m_live'])" >> $O/${TAG}_sweep.txt
}
for C in C5 C2; do
E=""; run; E="TC_CS_DIV=2"; run; E="TC_CS_DIV=4"; run; E="TC_SHORT_LINEAR=1"; run; E="TC_CS_DIV=2 TC_SHORT_LINEAR=1"; run
done
echo done > $O/${TAG}_done.txt
