TAG=${1:-r20j}
O=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sharded.py tests/test_gpu_support.py -q -x > $O/${TAG}_pytest.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest.txt
run() {
  env $E timeout 300 python bench.py --config $C --no-cpu-baseline --no-sharded --steps 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); b=d['build_ms']; print('$C $E', round(d['ms_per_step'],4), d['parity_vs_oracle'], 'build', round(b['total_events'],2), 'orient_csr', round(b['orient_csr'],2), 'e2e', round(d['e2e']['ms_per_step'],2))" >> $O/${TAG}_ab.txt
}
for C in C3 C2 C5 C1; do E=""; run; E="TC_A5=radix"; run; done
E=""; C=C4; timeout 1200 python bench.py --config C4 --no-cpu-baseline --no-sharded --steps 2 --e2e-steps 1 --out $O/${TAG}_bench_c4.json > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
