O=gpurun_out; T=r3a
BENCH_ARGS="--mode support" bash scripts/gpu_abbuild.sh ${T}c3 C3 5 "" "-DTC_SUP_L2PF=1" ""
BENCH_ARGS="--mode support" bash scripts/gpu_abbuild.sh ${T}c2 C2 10 "" "-DTC_SUP_L2PF=1"
echo done > $O/${T}_done.txt
