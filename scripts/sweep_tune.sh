# sweep the count kernel's launch tuning (TC_* env, tc_internal.cuh Tuning) on one config
cfg=${1:-C3}
for pd in 5 6 8 10; do for sl in 3 4; do
  r=$(TC_PROD_DIV=$pd TC_SLOTS=$sl timeout 200 python bench.py --config $cfg --no-cpu-baseline --no-e2e --steps 3 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['ms_per_step'],2), d['parity_vs_oracle'])")
  echo "prod_div=$pd slots=$sl -> $r"
done; done
