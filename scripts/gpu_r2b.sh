# r2b: measured-profile partition, robustness tests, sanitizers, bench C3.
O=gpurun_out; T=r2b
python -c "import bench; print(bench.src_hash())" > $O/${T}_src_hash.txt
timeout 1800 python -m pytest -q tests/test_gpu_balance.py tests/test_gpu_robust.py tests/test_gpu_fused.py -s > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
for tool in racecheck synccheck memcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python scripts/sanitize_case.py > $O/${T}_sanitize_${tool}.txt 2>&1; echo "rc=$?" >> $O/${T}_sanitize_${tool}.txt
done
timeout 900 python bench.py --steps 10 --warmup 3 --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
echo done > $O/${T}_done.txt
