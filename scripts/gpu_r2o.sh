O=gpurun_out; T=r2o
timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py -k "more_than" -s > $O/${T}_pytest_bigm.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest_bigm.txt
timeout 1800 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py tests/test_gpu_support.py > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${T}_launches_c3.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded --no-balance > /dev/null 2>&1
echo done > $O/${T}_done.txt
