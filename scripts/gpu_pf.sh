# A/B of the L2 bulk prefetch in the long-class producers + multicast probe
TAG=${1:-r19c}
O=gpurun_out
timeout 120 python scripts/probe_mc.py > $O/${TAG}_probe_mc.txt 2>&1
for pf in 0 1 0 1; do
  for c in C3 C2; do
    TC_PREFETCH=$pf timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c pf=$pf', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
  done
done
timeout 600 python -m pytest tests/test_gpu_sharded.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
echo done > $O/${TAG}_done.txt
