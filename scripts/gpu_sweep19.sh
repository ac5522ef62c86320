# sweep producer share / slots / wait hint on the current build (C3 count ms, parity)
TAG=${1:-r19i}
O=gpurun_out
run() {  # env-assignments...
  env "$@" timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['ms_per_step'],3), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt
}
run TC_PROD_DIV=8
run TC_PROD_DIV=6
run TC_PROD_DIV=5
run TC_PROD_DIV=4
run TC_PROD_DIV=8 TC_SLOTS=4
run TC_PROD_DIV=6 TC_SLOTS=4
run TC_PROD_DIV=8 TC_WAIT_HINT=2000
run TC_PROD_DIV=6 TC_WAIT_HINT=2000
run TC_PROD_DIV=8 TC_WAIT_HINT=20000
for c in C2 C5; do
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', round(d['ms_per_step'],4), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt
done
echo done > $O/${TAG}_done.txt
