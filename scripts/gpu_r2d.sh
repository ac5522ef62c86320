O=gpurun_out; T=r2d
TC_KEY_STAGES=3 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden" > $O/${T}_pytest_stages3.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest_stages3.txt
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_KEY_STAGES=2" "TC_KEY_STAGES=3" "TC_KEY_STAGES=4" "TC_KEY_STAGES=3 TC_PROD_DIV=4" ""
TC_KEY_STAGES=2 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 1 \
  -o $O/${T}_c3_stages2 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/${T}_ncu.log 2>&1
echo done > $O/${T}_done.txt
