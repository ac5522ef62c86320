TAG=${1:-r20h}
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > $O/${TAG}_pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_gpu.txt
for c in C1 C2 C5 C3; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --no-sharded --steps 10 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],4), d['parity_vs_oracle'], d['gpu_launches'])" >> $O/${TAG}_ab.txt
done
echo done > $O/${TAG}_done.txt
