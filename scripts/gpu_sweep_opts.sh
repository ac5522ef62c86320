# Plan-option sweep: bash scripts/gpu_sweep_opts.sh TAG "--opt a=1 --opt b=2" "..."
TAG=$1; shift
make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
OUT=gpurun_out/${TAG}_sweep.txt; : > $OUT
for o in "$@"; do
  for c in ${SWEEP_CONFIGS:-C3 C2 C5}; do
    timeout 240 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e $o --out /tmp/s.json > /dev/null 2>/tmp/s.err
    python -c "import json; d=json.load(open('/tmp/s.json')); print('$o', '$c', round(d['ms_per_step'],3), d['parity_vs_oracle'], d['plan']['n_chunks'], d['plan']['smem_bytes'])" >> $OUT 2>&1 || (echo "$o $c FAILED" >> $OUT; tail -3 /tmp/s.err >> $OUT)
  done
done
cat $OUT
