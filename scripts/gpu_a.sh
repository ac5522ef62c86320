set -x
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu3.txt 2>&1
timeout 300 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_c3_c.txt 2>&1
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-e2e > gpurun_out/bench_c2_c.txt 2>&1
timeout 300 python bench.py --config C5 --no-cpu-baseline --no-e2e > gpurun_out/bench_c5_c.txt 2>&1
