O=gpurun_out; T=r2l
timeout 1200 python scripts/diag_refine.py --config C4 --P 8 --slices 64,128,256 > $O/${T}_refine_c4.txt 2>&1
timeout 900 python scripts/diag_refine.py --config C3 --P 8 --slices 64,256 > $O/${T}_refine_c3.txt 2>&1
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_PROD_GROUPS=3 TC_PROD_DIV=3" "TC_PROD_GROUPS=2 TC_SLOTS=4" "TC_PROD_GROUPS=3 TC_PROD_DIV=3 TC_SLOTS=4" ""
timeout 600 python bench.py --config C5 --steps 10 --warmup 3 --no-cpu-baseline --out $O/${T}_c5.json > /dev/null 2>&1
echo done > $O/${T}_done.txt
