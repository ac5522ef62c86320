# One GPU pass: tests, C3/C2 bench lines, launch list + full ncu capture of the count kernel.
# usage: bash scripts/gpu_profile_c3.sh TAG
TAG=${1:-rX}
make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/${TAG}_pytest.txt
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_c3.json 2> gpurun_out/${TAG}_bench_c3.err
timeout 300 python bench.py --config C2 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_c2.json 2>&1
timeout 300 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench_c5.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_c3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/${TAG}_launch_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 -o gpurun_out/${TAG}_prof_c3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/${TAG}_ncu.log 2>&1
tail -2 gpurun_out/${TAG}_ncu.log
cat gpurun_out/${TAG}_pytest.txt | tail -3
