# C2 (short class) plan-option sweep: table load, bitmap threshold, chunk cost
TAG=${1:-r19n}
O=gpurun_out
run() {
  timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 10 "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C $*', round(d['ms_per_step'],4), d['parity_vs_oracle'], d['plan']['n_chunks'])" >> $O/${TAG}_sweep.txt
}
for C in C2 C5; do
run
run --opt table_factor=4
run --opt table_factor=6
run --opt bitmap_factor=8
run --opt bitmap_factor=16
run --opt chunk_cost=8192
run --opt chunk_cost=32768
run --opt probe_mode=1
done
C=C3; run --opt bitmap_factor=8; run --opt table_factor=4; run --opt chunk_cost=8192
echo done > $O/${TAG}_done.txt
