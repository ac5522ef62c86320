O=gpurun_out; T=r2z
bash scripts/gpu_abbuild.sh ${T}c3 C3 10 "" "-DTC_PF_ROWS=1" "-DTC_PF_FIRST=1" "-DTC_PF_ROWS=1 -DTC_PF_FIRST=1" ""
bash scripts/gpu_abbuild.sh ${T}c4 C4 3 "" "-DTC_PF_ROWS=1" "-DTC_PF_FIRST=1"
bash scripts/gpu_abbuild.sh ${T}c2 C2 20 "" "-DTC_PF_ROWS=1"
echo done > $O/${T}_done.txt
