TAG=${1:-r19o}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_support.py -q -x > $O/${TAG}_pytest_sup.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_sup.txt
timeout 600 python bench.py --mode support --no-sharded --out $O/${TAG}_bench_support_c3.json > /dev/null 2>&1
run() {
  env $E timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 10 "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C $E $*', round(d['ms_per_step'],4), d['parity_vs_oracle'], d['plan']['n_chunks'])" >> $O/${TAG}_sweep.txt
}
for C in C5 C2 C3; do
E=""; run
E="TC_CS_DIV=2"; run
E="TC_CS_DIV=4"; run
E=""; run --opt table_factor=6
E="TC_CS_DIV=2"; run --opt table_factor=6
E=""; run --opt table_factor=6 --opt bitmap_factor=8
E="TC_CS_DIV=2"; run --opt table_factor=6 --opt bitmap_factor=8
done
echo done > $O/${TAG}_done.txt
