# cp.async key ring (TC_RING=1) A/B: depth x slots x producer share, C3 count ms + parity
TAG=${1:-r19l}
O=gpurun_out
run() {
  env "$@" timeout 300 python bench.py --config C3 --no-cpu-baseline --no-e2e --no-sharded --steps 5 2>$O/${TAG}_err.txt | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('D=$D $*', round(d['ms_per_step'],3), d['parity_vs_oracle'], d['plan']['n_chunks'])" >> $O/${TAG}_sweep.txt || tail -3 $O/${TAG}_err.txt >> $O/${TAG}_sweep.txt
}
D=2
run TC_RING=0
run TC_RING=1 TC_SLOTS=3
run TC_RING=1 TC_SLOTS=2
run TC_RING=1 TC_SLOTS=2 TC_PROD_DIV=4
TC_RING=1 TC_SLOTS=2 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/${TAG}_pytest_ring.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_ring.txt
for D in 3 4; do
  touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="-DTC_RING_DEPTH=$D" > $O/${TAG}_make_$D.txt 2>&1
  run TC_RING=1 TC_SLOTS=3
  run TC_RING=1 TC_SLOTS=2
done
echo done > $O/${TAG}_done.txt
