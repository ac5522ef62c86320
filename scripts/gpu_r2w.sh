# The N > 1 bench path (agreed profile, ranges, sharded build, e2e, all_reduce) with
# 2 and 4 gloo ranks sharing cuda:0 -- a test of the code path, not a scaling number.
O=gpurun_out; T=r2w
for N in 2 4; do
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 \
    --master-port 2951$N bench.py --gpus $N --steps 3 --warmup 3 --config C2 --backend gloo --share-gpu \
    --out $O/${T}_bench_c2_n$N.json > $O/${T}_bench_c2_n$N.log 2>&1; echo "rc=$?" >> $O/${T}_bench_c2_n$N.log
done
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29520 bench.py --gpus 2 --steps 3 --warmup 3 --e2e-steps 1 --config C3 --backend gloo --share-gpu \
  --out $O/${T}_bench_c3_n2.json > $O/${T}_bench_c3_n2.log 2>&1; echo "rc=$?" >> $O/${T}_bench_c3_n2.log
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29530 bench.py --gpus 2 --impl reference --steps 2 --warmup 1 --config C2 \
  --out $O/${T}_reference_c2_n2.json > $O/${T}_reference_c2_n2.log 2>&1; echo "rc=$?" >> $O/${T}_reference_c2_n2.log
echo done > $O/${T}_done.txt
