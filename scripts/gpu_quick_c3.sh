# Quick pass: C3 bench (no cpu baseline / e2e), plan trace, ncu capture.  usage: bash scripts/gpu_quick_c3.sh TAG
TAG=${1:-q}
make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
TC_VERBOSE=1 timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_c3.json 2> gpurun_out/${TAG}_bench_c3.err
timeout 300 python bench.py --config C2 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${TAG}_bench_c2.json 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 -o gpurun_out/${TAG}_prof_c3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/${TAG}_ncu.log 2>&1
tail -1 gpurun_out/${TAG}_ncu.log
