# Regenerate the committed evidence of one tree on one B200 (run under gpurun):
#   bash scripts/gpu_evidence.sh TAG
# then, here: python scripts/profile_summary.py gpurun_out/TAG_c3_count.ncu-rep TAG C3 \
#               --src-hash $(cat gpurun_out/TAG_src_hash.txt)   (and C2), and copy the rest
# into profiles/ (scripts/collect_evidence.py TAG).
T=${1:?tag}; O=gpurun_out
python -c "import bench; print(bench.src_hash())" > $O/${T}_src_hash.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/${T}_smi.txt
timeout 2400 python -m pytest tests -m gpu -q > $O/${T}_pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${T}_smoke.txt 2>&1; echo "rc=$?" >> $O/${T}_smoke.txt
timeout 900 python bench.py --steps 20 --warmup 5 --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
for c in C1 C2 C5; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 5 --out $O/${T}_bench_$(echo $c | tr C c).json > $O/${T}_bench_$c.log 2>&1
done
timeout 1800 python bench.py --config C4 --steps 3 --warmup 3 --no-cpu-baseline --no-sharded --e2e-steps 1 --out $O/${T}_bench_c4.json > $O/${T}_bench_c4.log 2>&1
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 --out $O/${T}_reference_c3.json > $O/${T}_reference_c3.log 2>&1
for c in C3 C2; do
  timeout 900 python bench.py --config $c --mode support --steps 5 --warmup 3 --out $O/${T}_bench_support_$(echo $c | tr C c).json > $O/${T}_bench_support_$c.log 2>&1
done
for v in polak trust; do for c in C1 C2 C5 C3; do
  timeout 900 python bench.py --config $c --variant $v --steps 3 --warmup 3 --no-e2e --no-sharded --no-cpu-baseline \
    --no-balance --out $O/${T}_bench_${v}_$(echo $c | tr C c).json > $O/${T}_bench_${v}_$c.log 2>&1
done; done
timeout 1800 python scripts/oracle_times.py > $O/${T}_oracle_times.jsonl 2> $O/${T}_oracle_times.err
# (compute-sanitizer is closed on the gpurun pool since r4a; the r2b / r2j logs are the last runs:
#  for tool in racecheck synccheck memcheck: compute-sanitizer --tool $tool python scripts/sanitize_case.py)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${T}_launches_c3.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded --no-balance > $O/${T}_launches.log 2>&1
for c in C3 C2; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 2 \
    -o $O/${T}_$(echo $c | tr C c)_count python bench.py --config $c --steps 1 --warmup 1 --no-cpu-baseline --no-e2e \
    --no-sharded --no-balance > $O/${T}_ncu_$c.log 2>&1
done
echo done > $O/${T}_done.txt
