# Round evidence on one B200: GPU tests, bench lines, launch list, ncu captures.
# usage: bash scripts/gpu_round.sh TAG   (outputs under gpurun_out/TAG_*)
TAG=${1:-r19}
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $O/${TAG}_smi.txt
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_gpu.txt
timeout 600 python bench.py --out $O/${TAG}_bench_c3.json > $O/${TAG}_bench_c3.log 2>&1
for c in C1 C2 C5; do timeout 400 python bench.py --config $c --out $O/${TAG}_bench_$(echo $c | tr A-Z a-z).json > /dev/null 2>&1; done
timeout 1200 python bench.py --config C4 --no-cpu-baseline --no-sharded --steps 3 --e2e-steps 1 --out $O/${TAG}_bench_c4.json > $O/${TAG}_bench_c4.log 2>&1
timeout 600 python bench.py --mode support --out $O/${TAG}_bench_support_c3.json > /dev/null 2>&1
for c in C1 C5; do timeout 300 python bench.py --config $c --reduce fused --no-cpu-baseline --no-e2e --no-sharded --steps 20 --out $O/${TAG}_bench_fused_$(echo $c | tr A-Z a-z).json > /dev/null 2>&1; done
for v in polak trust; do for c in C1 C2 C3 C5; do
  timeout 600 python bench.py --config $c --variant $v --no-cpu-baseline --no-e2e --no-sharded --steps 3 --out $O/${TAG}_bench_${v}_$(echo $c | tr A-Z a-z).json > /dev/null 2>&1
done; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 --out $O/${TAG}_reference_c3.json > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${TAG}_launches_c3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_count$" -s 1 -c 1 -o $O/${TAG}_prof_c3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_count_flat" -s 1 -c 1 -o $O/${TAG}_prof_c3_flat python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_support" -s 1 -c 1 -o $O/${TAG}_prof_support_c3 python bench.py --mode support --steps 1 --warmup 1 --no-cpu-baseline --no-sharded > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
