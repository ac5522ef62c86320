# support parity tests + default support bench lines after TC_UNROLL_SUP 6 -> 5
TAG=${1:-r24v}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_support.py -q -x > $O/${TAG}_pytest_support.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_support.txt
timeout 600 python bench.py --mode support --no-sharded --out $O/${TAG}_bench_support_c3.json > /dev/null 2>&1
timeout 600 python bench.py --mode support --config C2 --no-sharded --out $O/${TAG}_bench_support_c2.json > /dev/null 2>&1
timeout 600 python bench.py --mode support --config C5 --no-sharded --out $O/${TAG}_bench_support_c5.json > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
