O=gpurun_out; T=r2n
timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py -k "a5_paths or csr_exact or host_pipelined or full_size or closed_forms or more_than" > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
TC_A5=sort timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-balance --out $O/${T}_bench_c3_a5sort.json > $O/${T}_bench_c3_a5sort.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${T}_launches_c3.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded --no-balance > /dev/null 2>&1
echo done > $O/${T}_done.txt
