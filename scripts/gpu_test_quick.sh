# GPU tests + quick C3/C2/C5 bench (no ncu).  usage: bash scripts/gpu_test_quick.sh TAG
TAG=${1:-t}
make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -15 > gpurun_out/${TAG}_pytest.txt
tail -3 gpurun_out/${TAG}_pytest.txt
for c in C3 C2 C5; do
  TC_VERBOSE=1 timeout 180 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_${c}.json 2> gpurun_out/${TAG}_bench_${c}.err
done
