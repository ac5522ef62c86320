TAG=${1:-r19p}
O=gpurun_out
run() {
  env $E timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 10 "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C $E $*', round(d['ms_per_step'],4), d['parity_vs_oracle'], d['plan']['n_chunks'])" >> $O/${TAG}_sweep.txt
}
for C in C5 C2 C3; do
E=""; run --opt table_factor=6 --opt bitmap_factor=8
E="TC_SHORT_LINEAR=1"; run --opt table_factor=6 --opt bitmap_factor=8
E="TC_SHORT_LINEAR=1"; run --opt table_factor=4 --opt bitmap_factor=8
E=""; run --opt table_factor=8 --opt bitmap_factor=8
E=""; run --opt table_factor=6 --opt bitmap_factor=12
E=""; run --opt table_factor=6 --opt bitmap_factor=16
done
echo done > $O/${TAG}_done.txt
