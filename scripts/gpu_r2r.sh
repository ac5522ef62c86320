O=gpurun_out; T=r2r
timeout 1800 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_support.py tests/test_gpu_fused.py > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
bash scripts/gpu_ab.sh ${T}c2 C2 20 "" "BENCH_OPT=bitmap_factor=12"
bash scripts/gpu_ab.sh ${T}c5 C5 20 "" "BENCH_OPT=bitmap_factor=12"
bash scripts/gpu_ab.sh ${T}c1 C1 20 "" "BENCH_OPT=bitmap_factor=12"
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
echo done > $O/${T}_done.txt
