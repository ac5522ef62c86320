# r2a: new partition / fused / roofline code on the B200 + L2-policy A/B at C3.
O=gpurun_out; T=r2a
python -c "import bench; print(bench.src_hash())" > $O/${T}_src_hash.txt
timeout 1500 python -m pytest -q tests/test_gpu_fused.py tests/test_gpu_balance.py \
  "tests/test_gpu_parity.py::test_full_size_vs_stored_oracle" "tests/test_gpu_parity.py::test_partition_ranges_sum_to_total" \
  tests/test_gpu_parity.py::test_c1_rmat10_seeds -s > $O/${T}_pytest.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest.txt
timeout 600 python bench.py --steps 10 --warmup 3 --out $O/${T}_bench_c3.json > $O/${T}_bench_c3.log 2>&1
for kv in "TC_L2_META=1" "TC_L2_KEYS=2" "TC_L2_KEYS=1" "TC_L2_PERSIST_MB=80" "TC_L2_META=1 TC_L2_PERSIST_MB=80" ; do
  tag=$(echo $kv | tr ' =' '__')
  env $kv timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-sharded --no-cpu-baseline --no-balance --out $O/${T}_ab_${tag}.json > $O/${T}_ab_${tag}.log 2>&1
done
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-sharded --no-cpu-baseline --no-balance --out $O/${T}_ab_base2.json > $O/${T}_ab_base2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 2 \
  -o $O/${T}_c3_count python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/${T}_ncu.log 2>&1
echo done > $O/${T}_done.txt
