# Round-2 first look: device attributes, per-range balance at C3, ncu of k_count.
O=gpurun_out
python - <<'PY' > $O/d1_attrs.txt 2>&1
from cuda.bindings import runtime as rt
for a in ["cudaDevAttrMaxPersistingL2CacheSize", "cudaDevAttrL2CacheSize", "cudaDevAttrMaxAccessPolicyWindowSize"]:
    print(a, rt.cudaDeviceGetAttribute(getattr(rt.cudaDeviceAttr, a), 0))
PY
timeout 900 python scripts/diag_balance.py --config C3 > $O/d1_balance_c3.txt 2>&1
timeout 900 python scripts/diag_balance.py --config C2 > $O/d1_balance_c2.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 2 \
  -o $O/d1_c3_count python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded > $O/d1_ncu.log 2>&1
echo done > $O/d1_done.txt
