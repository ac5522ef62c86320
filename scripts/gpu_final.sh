# final check of the committed tree: GPU suite, smoke(), default bench line
TAG=${1:-r22}
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_pytest_gpu.txt 2>&1; echo "rc=$?" >> $O/${TAG}_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.txt 2>&1; echo "rc=$?" >> $O/${TAG}_smoke.txt
timeout 900 python bench.py --out $O/${TAG}_bench_c3.json > $O/${TAG}_bench_c3.log 2>&1
timeout 900 python bench.py --impl reference --out $O/${TAG}_reference_c3.json > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
timeout 600 python bench.py --mode support --no-sharded --out $O/${TAG}_bench_support_c3.json > /dev/null 2>&1
timeout 600 python bench.py --mode support --config C2 --no-sharded --out $O/${TAG}_bench_support_c2.json > /dev/null 2>&1
echo done2 >> $O/${TAG}_done.txt
