O=gpurun_out; T=r2y
bash scripts/gpu_abbuild.sh ${T}c2 C2 20 "" "-DTC_PF_SHORT=1" ""
bash scripts/gpu_abbuild.sh ${T}c3 C3 10 "" "-DTC_PF_SHORT=1"
bash scripts/gpu_abbuild.sh ${T}c5 C5 20 "" "-DTC_PF_SHORT=1"
echo done > $O/${T}_done.txt
