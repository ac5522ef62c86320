# A/B of count-kernel knobs on ONE box: bench.py (count step only) per setting.
#   bash scripts/gpu_ab.sh TAG CONFIG STEPS "ENV1" "ENV2" ...   ("" = defaults)
# Writes gpurun_out/TAG_ab_<i>.json/.log and TAG_ab.txt (one line per setting).
T=$1; CFG=$2; STEPS=$3; shift 3
O=gpurun_out; i=0
for kv in "$@"; do
  env $kv timeout 600 python bench.py --config $CFG --steps $STEPS --warmup 3 --no-e2e --no-sharded \
    --no-cpu-baseline --no-balance --out $O/${T}_ab_$i.json > $O/${T}_ab_$i.log 2>&1
  python - "$O/${T}_ab_$i.json" "$kv" >> $O/${T}_ab.txt <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[1])); r = d["roofline"]
    print(f"{sys.argv[2] or 'default':36s} step {d['ms_per_step']:8.3f} ms  k_count {r['kernel_ms']:8.3f} ms  "
          f"frac {r['frac']:.3f}  parity {d['parity_vs_oracle']}  T {d['triangles']}")
except Exception as e:
    print(f"{sys.argv[2] or 'default':36s} FAILED {e!r}")
PY
  i=$((i+1))
done
