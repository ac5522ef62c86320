TAG=${1:-r20b}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "host or csr_exact or dedup" > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
timeout 600 python bench.py --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c3.json > /dev/null 2>&1
TC_H2D_PIECES=2 timeout 600 python bench.py --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c3_p2.json > /dev/null 2>&1
TC_H2D_PIECES=8 timeout 600 python bench.py --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c3_p8.json > /dev/null 2>&1
TC_H2D_PIECES=1 timeout 600 python bench.py --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c3_p1.json > /dev/null 2>&1
timeout 1200 python bench.py --config C4 --no-cpu-baseline --no-sharded --steps 3 --e2e-steps 2 --out $O/${TAG}_bench_c4.json > $O/${TAG}_bench_c4.log 2>&1
echo done > $O/${TAG}_done.txt
