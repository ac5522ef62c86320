O=gpurun_out; T=r2f
timeout 600 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or full_size" > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
bash scripts/gpu_ab.sh ${T} C3 10 "" \
  "BENCH_OPT=block_threads=768" "BENCH_OPT=block_threads=768 TC_BATCH=12" "BENCH_OPT=block_threads=768 TC_BATCH=16" \
  "BENCH_OPT=block_threads=768 TC_BATCH=12 TC_PROD_DIV=4" "BENCH_OPT=block_threads=512 TC_BATCH=16 TC_PROD_DIV=4" \
  "BENCH_OPT=block_threads=512 TC_BATCH=24 TC_PROD_DIV=4" "BENCH_OPT=block_threads=512 TC_BATCH=16" ""
echo done > $O/${T}_done.txt
