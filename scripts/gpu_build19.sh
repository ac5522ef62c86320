# k_split fast path + hash dedup: parity tests and build timings
TAG=${1:-r19k}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharded.py tests/test_gpu_support.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
for c in C3 C2 C5 C1; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_$(echo $c | tr A-Z a-z).json > /dev/null 2>&1
done
TC_DEDUP=sort timeout 300 python bench.py --config C3 --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c3_sortdedup.json > /dev/null 2>&1
timeout 1200 python bench.py --config C4 --no-cpu-baseline --no-sharded --steps 3 --e2e-steps 1 --out $O/${TAG}_bench_c4.json > $O/${TAG}_bench_c4.log 2>&1
echo done > $O/${TAG}_done.txt
