O=gpurun_out; T=r2k
for kv in "TC_PROD_GROUPS=2" "TC_PIPE=1"; do
  env $kv timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or partition" > $O/${T}_pytest_$(echo $kv | tr '=' '_').txt 2>&1; echo "rc=$?" >> $O/${T}_pytest_$(echo $kv | tr '=' '_').txt
done
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_PROD_GROUPS=2" "TC_PIPE=1" "TC_PROD_GROUPS=2 TC_PIPE=1" "TC_PROD_GROUPS=2 TC_PROD_DIV=3" "TC_PROD_GROUPS=2 TC_PROD_DIV=5" ""
bash scripts/gpu_ab.sh ${T}c4 C4 3 "" "TC_PROD_GROUPS=2" "TC_PIPE=1"
echo done > $O/${T}_done.txt
timeout 900 python -m pytest -q tests/test_gpu_balance.py -s > $O/${T}_balance1.txt 2>&1
timeout 900 python -m pytest -q tests/test_gpu_balance.py -s > $O/${T}_balance2.txt 2>&1
timeout 600 python bench.py --config C5 --steps 10 --warmup 3 --no-cpu-baseline --out $O/${T}_c5_bal.json > /dev/null 2>&1
timeout 600 python bench.py --config C5 --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/${T}_c5_nobal.json > /dev/null 2>&1
