O=gpurun_out; T=r2t
TC_HOSTTIME=1 timeout 600 python scripts/diag_e2e.py C3 10 > $O/${T}_e2e_c3.txt 2>&1
echo done > $O/${T}_done.txt
