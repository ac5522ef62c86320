# f4 fused sum + f2 sharded: GPU tests, C1/C2/C3 bench with --reduce fused vs nccl
TAG=${1:-r19d}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_fused.py tests/test_gpu_sharded.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
for r in nccl fused; do for c in C1 C5 C3; do
  timeout 300 python bench.py --config $c --reduce $r --no-cpu-baseline --no-e2e --no-sharded --steps 20 --out $O/${TAG}_bench_${r}_$(echo $c | tr A-Z a-z).json > /dev/null 2>&1
done; done
echo done > $O/${TAG}_done.txt
