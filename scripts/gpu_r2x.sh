O=gpurun_out; T=r2x
bash scripts/gpu_abbuild.sh ${T}c3 C3 10 "" "-DTC_L2PF=2" "-DTC_L2PF=3" "-DTC_PF_NEXT=1" "-DTC_L2PF=2 -DTC_PF_NEXT=1" ""
bash scripts/gpu_abbuild.sh ${T}c4 C4 3 "" "-DTC_L2PF=2" "-DTC_PF_NEXT=1"
echo done > $O/${T}_done.txt
