# f2 sharded build: GPU tests + bench lines with the sharded-build measurement.
TAG=${1:-r19b}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_parity.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
timeout 600 python bench.py --no-cpu-baseline --out $O/${TAG}_bench_c3.json > $O/${TAG}_bench_c3.log 2>&1
timeout 300 python bench.py --config C2 --no-cpu-baseline --out $O/${TAG}_bench_c2.json > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
