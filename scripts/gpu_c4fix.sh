TAG=${1:-r21b}
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_support.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
for c in C3 C2 C5; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],4), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
done
timeout 1500 python bench.py --config C4 --no-cpu-baseline --no-sharded --steps 3 --e2e-steps 1 --out $O/${TAG}_bench_c4.json > $O/${TAG}_bench_c4.log 2>&1
echo done > $O/${TAG}_done.txt
