O=gpurun_out; T=r3b
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_PROD_DIV=3" "TC_PROD_DIV=5" "TC_PROD_DIV=3 TC_PROD_GROUPS=3" "TC_SLOTS=4" "TC_SLOTS=2" ""
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 2 \
  -o $O/${T}_c3_count python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/${T}_ncu.log 2>&1
python -c "import bench; print(bench.src_hash())" > $O/${T}_src_hash.txt
echo done > $O/${T}_done.txt
