O=gpurun_out; T=r2h
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_PROD_DIV=4" "TC_PROD_DIV=3" "TC_PROD_DIV=4 TC_SLOTS=4" "TC_PROD_DIV=4 TC_SLOTS=2" "TC_PROD_DIV=4" ""
bash scripts/gpu_ab.sh ${T}c4 C4 3 "" "TC_PROD_DIV=4" "TC_PROD_DIV=3"
echo done > $O/${T}_done.txt
