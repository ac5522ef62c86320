O=gpurun_out; T=r2e
bash scripts/gpu_ab.sh ${T}c3 C3 10 "" "BENCH_OPT=long_min=48" "BENCH_OPT=long_min=64" "BENCH_OPT=long_min=96" "BENCH_OPT=long_min=128" ""
bash scripts/gpu_ab.sh ${T}c2 C2 20 "" "BENCH_OPT=long_min=64" "BENCH_OPT=long_min=128"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 \
  -o $O/${T}_c3_head5 python scripts/profile_range.py --config C3 --lo 0 --hi 0.05 > $O/${T}_ncu_head5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 \
  -o $O/${T}_c3_mid python scripts/profile_range.py --config C3 --lo 0.45 --hi 0.55 > $O/${T}_ncu_mid.log 2>&1
echo done > $O/${T}_done.txt
