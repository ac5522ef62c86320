# A/B of compile-time knobs on ONE box: rebuild libtc.so with NVEXTRA per setting,
# run bench.py (count step only), restore the default build at the end.
#   bash scripts/gpu_abbuild.sh TAG CONFIG STEPS "-DX=1" "-DX=2" ...   ("" = defaults)
T=$1; CFG=$2; STEPS=$3; shift 3
O=gpurun_out; i=0
for fl in "$@"; do
  rm -f build/tc_count.o paper_conf_ipps_li0ptz24_b200/libtc.so
  make -s NVEXTRA="$fl" paper_conf_ipps_li0ptz24_b200/libtc.so > $O/${T}_build_$i.log 2>&1
  timeout 600 python bench.py --config $CFG --steps $STEPS --warmup 3 --no-e2e --no-sharded $BENCH_ARGS \
    --no-cpu-baseline --no-balance --out $O/${T}_ab_$i.json > $O/${T}_ab_$i.log 2>&1
  python - "$O/${T}_ab_$i.json" "$fl" >> $O/${T}_ab.txt <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[1])); r = d["roofline"]
    print(f"{sys.argv[2] or 'default':36s} step {d['ms_per_step']:8.3f} ms  {r.get('kernel', 'support')[:12]} {r.get('kernel_ms', d['ms_per_step']):8.3f} ms  "
          f"frac {r['frac']:.3f}  parity {d['parity_vs_oracle']}  T {d['triangles']}")
except Exception as e:
    print(f"{sys.argv[2] or 'default':36s} FAILED {e!r}")
PY
  i=$((i+1))
done
rm -f build/tc_count.o paper_conf_ipps_li0ptz24_b200/libtc.so
make -s paper_conf_ipps_li0ptz24_b200/libtc.so > /dev/null 2>&1
