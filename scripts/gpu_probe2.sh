TAG=${1:-r19f}
O=gpurun_out
timeout 120 python scripts/probe_mc2.py > $O/${TAG}_probe_mc2.txt 2>&1
ls /dev/nvidia* >> $O/${TAG}_probe_mc2.txt 2>&1
nvidia-smi -q | grep -i -A3 "fabric" >> $O/${TAG}_probe_mc2.txt 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x > $O/${TAG}_pytest_parity.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_parity.txt
for c in C3 C2 C3 C5; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_ab.txt
done
echo done > $O/${TAG}_done.txt
