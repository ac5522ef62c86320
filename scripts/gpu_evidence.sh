# Full evidence pass for profiles/: GPU tests, bench lines (C3 with cpu_baseline + e2e; C1/C2/C5),
# launch list of the C3 bench command, ncu --set full of both count kernels at C3.
# usage: bash scripts/gpu_evidence.sh TAG
TAG=${1:-ev}
make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -5 > gpurun_out/${TAG}_pytest.txt
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_c3.json 2> gpurun_out/${TAG}_bench_c3.err
for c in C1 C2 C5; do
  lc=$(echo $c | tr 'A-Z' 'a-z')
  timeout 300 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_${lc}.json 2> gpurun_out/${TAG}_bench_${lc}.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_reference_c3.json 2> gpurun_out/${TAG}_reference_c3.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches_c3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/${TAG}_launch_run.log 2>&1
K="k_count k_count_flat" bash scripts/gpu_ncu.sh ${TAG} C3
tail -3 gpurun_out/${TAG}_pytest.txt
