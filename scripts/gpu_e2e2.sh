TAG=${1:-r20c}
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
for i in 1 2; do
timeout 600 python bench.py --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c3_$i.json > /dev/null 2>&1
done
timeout 300 python bench.py --config C2 --no-cpu-baseline --no-sharded --steps 5 --out $O/${TAG}_bench_c2.json > /dev/null 2>&1
for p in 1 8; do
TC_H2D_PIECES=$p timeout 1200 python bench.py --config C4 --no-cpu-baseline --no-sharded --steps 2 --e2e-steps 2 --out $O/${TAG}_bench_c4_p$p.json > /dev/null 2>&1
done
echo done > $O/${TAG}_done.txt
