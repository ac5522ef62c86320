O=gpurun_out; T=r2q
TC_OVERLAP=1 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or partition or full_size" > $O/${T}_pytest_overlap.txt 2>&1; echo "rc=$?" >> $O/${T}_pytest_overlap.txt
bash scripts/gpu_ab.sh ${T} C3 10 "" "TC_OVERLAP=1" "BENCH_OPT=bitmap_factor=16" "BENCH_OPT=bitmap_factor=24" "BENCH_OPT=bitmap_factor=32" "TC_OVERLAP=1 BENCH_OPT=bitmap_factor=24" ""
bash scripts/gpu_ab.sh ${T}c4 C4 3 "" "TC_OVERLAP=1" "BENCH_OPT=bitmap_factor=24"
bash scripts/gpu_ab.sh ${T}c2 C2 20 "" "TC_OVERLAP=1"
echo done > $O/${T}_done.txt
