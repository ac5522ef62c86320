O=gpurun_out; T=r2u
bash scripts/gpu_abbuild.sh ${T}c2 C2 20 "" "-DTC_UNROLL_SHORT=3" "-DTC_UNROLL_SHORT=4" ""
bash scripts/gpu_abbuild.sh ${T}c3 C3 10 "" "-DTC_UNROLL_SHORT=3" "-DTC_UNROLL_SHORT=4"
bash scripts/gpu_abbuild.sh ${T}c5 C5 20 "" "-DTC_UNROLL_SHORT=3" "-DTC_UNROLL_SHORT=4"
echo done > $O/${T}_done.txt
