O=gpurun_out; T=r2s
timeout 600 python scripts/diag_e2e.py C3 12 > $O/${T}_e2e_c3.txt 2>&1
TC_H2D_PIECES=4 timeout 600 python scripts/diag_e2e.py C3 6 > $O/${T}_e2e_c3_p4.txt 2>&1
echo done > $O/${T}_done.txt
