TAG=${1:-r20g}
O=gpurun_out
run() {
  timeout 300 python bench.py --config $C --no-cpu-baseline --no-e2e --no-sharded --steps 10 "$@" 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$V $C $*', round(d['ms_per_step'],4), d['parity_vs_oracle'])" >> $O/${TAG}_sweep.txt
}
V=default; C=C1; run; run --opt long_min=1073741824; C=C5; run --opt long_min=1073741824
for cfg in "384 4 2" "320 5 4" "352 4 4"; do
  set -- $cfg
  V="block=$1 ctas=$2 unroll=$3"
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_FLAT_BLOCK=$1 -DTC_FLAT_CTAS=$2 -DTC_UNROLL_SHORT=$3" > $O/${TAG}_make.txt 2>&1
  for C in C2 C5 C3; do run; done
done
touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
echo done > $O/${TAG}_done.txt
