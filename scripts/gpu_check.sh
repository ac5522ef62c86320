# Re-entry check on one B200: the full GPU test suite and the default bench line.
TAG=${1:-r19}
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/${TAG}_smi.txt
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_gpu.txt
timeout 600 python bench.py --out $O/${TAG}_bench_c3.json > $O/${TAG}_bench_c3.log 2>&1
echo done > $O/${TAG}_done.txt
