# f4 multicast retry + address-arithmetic change of walk_long (C3/C2 timing + parity)
TAG=${1:-r19e}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_fused.py tests/test_gpu_sharded.py -q > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/${TAG}_pytest_parity.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_parity.txt
for c in C3 C2 C3; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
done
timeout 300 python bench.py --config C1 --reduce fused --no-cpu-baseline --no-e2e --no-sharded --steps 20 --out $O/${TAG}_bench_fused_c1.json > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
