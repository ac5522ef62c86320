# quick correctness + C3/C2 count timing (used while iterating on the count kernel)
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_quick.txt 2>&1
for c in C3 C2; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> gpurun_out/quick.txt
done
