TAG=${1:-r22b}
O=gpurun_out
run() {
  env $E timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C $E', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
}
for C in C3 C4; do E="TC_INTERLEAVE=0"; run; E="TC_INTERLEAVE=1"; run; E="TC_INTERLEAVE=1 TC_PROD_DIV=6"; run; E="TC_INTERLEAVE=1 TC_PROD_DIV=4"; run; done
C=C2; E="TC_INTERLEAVE=0"; run; E="TC_INTERLEAVE=1"; run
TC_INTERLEAVE=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "partition or ranges or config or full_size or rmat" > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
echo done > $O/${TAG}_done.txt
