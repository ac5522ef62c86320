make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -15 > gpurun_out/r2_pytest.txt
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench_c3.json 2> gpurun_out/r2_bench_c3.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2_launches_c3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2_launch_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 -o gpurun_out/r2_prof_c3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/r2_ncu.log 2>&1
tail -3 gpurun_out/r2_ncu.log
