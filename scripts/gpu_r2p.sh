O=gpurun_out; T=r2p
bash scripts/gpu_ab.sh ${T} C3 10 "" "BENCH_OPT=bitmap_factor=8" "BENCH_OPT=bitmap_factor=20" "BENCH_OPT=table_factor=4" "BENCH_OPT=table_factor=8" \
  "BENCH_OPT=chunk_cost=12288" "BENCH_OPT=chunk_cost=24576" "BENCH_OPT=seg_cost=2" "BENCH_OPT=seg_cost=8" ""
bash scripts/gpu_ab.sh ${T}c2 C2 20 "" "BENCH_OPT=table_factor=4" "BENCH_OPT=table_factor=8" "BENCH_OPT=chunk_cost=8192" "BENCH_OPT=chunk_cost=24576" ""
echo done > $O/${T}_done.txt
