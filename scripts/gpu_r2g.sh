O=gpurun_out; T=r2g
timeout 1200 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_PROD_DIV=4" \
  "BENCH_OPT=block_threads=768 TC_BATCH=8 TC_PROD_DIV=4" "BENCH_OPT=block_threads=768 TC_BATCH=12 TC_PROD_DIV=4" \
  "BENCH_OPT=block_threads=768 TC_BATCH=16 TC_PROD_DIV=4" "BENCH_OPT=block_threads=768 TC_BATCH=12 TC_PROD_DIV=3" ""
for c in C2 C5 C1; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-balance --out $O/${T}_bench_$(echo $c | tr C c).json > $O/${T}_bench_$c.log 2>&1; done
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
echo done > $O/${T}_done.txt
