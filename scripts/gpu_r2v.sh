O=gpurun_out; T=r2v
bash scripts/gpu_abbuild.sh ${T}c3 C3 10 "" "-DTC_L2PF=1" "" "-DTC_L2PF=1"
bash scripts/gpu_abbuild.sh ${T}c4 C4 3 "" "-DTC_L2PF=1"
echo done > $O/${T}_done.txt
