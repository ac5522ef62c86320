# Every A/B run of round 2, by tag (their outputs are profiles/<tag>_*).
#   bash scripts/ab_runs.sh TAG      (under gpurun; writes gpurun_out/TAG_*)
# Each run uses gpu_ab.sh (runtime env knobs) or gpu_abbuild.sh (compile-time -D knobs).
# Several knobs named here were removed after their A/B (DESIGN.md §6.2 table); the case bodies record
# what was run, against the tree of that commit.
T=${1:?tag}; O=gpurun_out
case "$T" in
r2a)
  # r2a: new partition / fused / roofline code on the B200 + L2-policy A/B at C3.
  python -c "import bench; print(bench.src_hash())" > $O/r2a_src_hash.txt
  timeout 1500 python -m pytest -q tests/test_gpu_fused.py tests/test_gpu_balance.py \
    "tests/test_gpu_parity.py::test_full_size_vs_stored_oracle" "tests/test_gpu_parity.py::test_partition_ranges_sum_to_total" \
    tests/test_gpu_parity.py::test_c1_rmat10_seeds -s > $O/r2a_pytest.txt 2>&1; echo "rc=$?" >> $O/r2a_pytest.txt
  timeout 600 python bench.py --steps 10 --warmup 3 --out $O/r2a_bench_c3.json > $O/r2a_bench_c3.log 2>&1
  for kv in "TC_L2_META=1" "TC_L2_KEYS=2" "TC_L2_KEYS=1" "TC_L2_PERSIST_MB=80" "TC_L2_META=1 TC_L2_PERSIST_MB=80" ; do
    tag=$(echo $kv | tr ' =' '__')
    env $kv timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-sharded --no-cpu-baseline --no-balance --out $O/r2a_ab_${tag}.json > $O/r2a_ab_${tag}.log 2>&1
  done
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-sharded --no-cpu-baseline --no-balance --out $O/r2a_ab_base2.json > $O/r2a_ab_base2.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 2 \
    -o $O/r2a_c3_count python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/r2a_ncu.log 2>&1
  ;;
r2b)
  # r2b: measured-profile partition, robustness tests, sanitizers, bench C3.
  python -c "import bench; print(bench.src_hash())" > $O/r2b_src_hash.txt
  timeout 1800 python -m pytest -q tests/test_gpu_balance.py tests/test_gpu_robust.py tests/test_gpu_fused.py -s > $O/r2b_pytest.txt 2>&1; echo "rc=$?" >> $O/r2b_pytest.txt
  for tool in racecheck synccheck memcheck; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 50 python scripts/sanitize_case.py > $O/r2b_sanitize_${tool}.txt 2>&1; echo "rc=$?" >> $O/r2b_sanitize_${tool}.txt
  done
  timeout 900 python bench.py --steps 10 --warmup 3 --out $O/r2b_bench_c3.json > $O/r2b_bench_c3.log 2>&1
  ;;
r2c)
  TC_KEY_STAGES=3 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden" > $O/r2c_pytest_stages3.txt 2>&1; echo "rc=$?" >> $O/r2c_pytest_stages3.txt
  bash scripts/gpu_ab.sh r2c C3 10 "" "TC_KEY_STAGES=2" "TC_KEY_STAGES=3" "TC_KEY_STAGES=4" ""
  TC_KEY_STAGES=3 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 1 \
    -o $O/r2c_c3_stages3 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/r2c_ncu.log 2>&1
  ;;
r2d)
  TC_KEY_STAGES=3 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden" > $O/r2d_pytest_stages3.txt 2>&1; echo "rc=$?" >> $O/r2d_pytest_stages3.txt
  bash scripts/gpu_ab.sh r2d C3 10 "" "TC_KEY_STAGES=2" "TC_KEY_STAGES=3" "TC_KEY_STAGES=4" "TC_KEY_STAGES=3 TC_PROD_DIV=4" ""
  TC_KEY_STAGES=2 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 1 \
    -o $O/r2d_c3_stages2 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/r2d_ncu.log 2>&1
  ;;
r2e)
  bash scripts/gpu_ab.sh r2ec3 C3 10 "" "BENCH_OPT=long_min=48" "BENCH_OPT=long_min=64" "BENCH_OPT=long_min=96" "BENCH_OPT=long_min=128" ""
  bash scripts/gpu_ab.sh r2ec2 C2 20 "" "BENCH_OPT=long_min=64" "BENCH_OPT=long_min=128"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 \
    -o $O/r2e_c3_head5 python scripts/profile_range.py --config C3 --lo 0 --hi 0.05 > $O/r2e_ncu_head5.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 1 -c 1 \
    -o $O/r2e_c3_mid python scripts/profile_range.py --config C3 --lo 0.45 --hi 0.55 > $O/r2e_ncu_mid.log 2>&1
  ;;
r2f)
  timeout 600 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or full_size" > $O/r2f_pytest.txt 2>&1; echo "rc=$?" >> $O/r2f_pytest.txt
  bash scripts/gpu_ab.sh r2f C3 10 "" \
    "BENCH_OPT=block_threads=768" "BENCH_OPT=block_threads=768 TC_BATCH=12" "BENCH_OPT=block_threads=768 TC_BATCH=16" \
    "BENCH_OPT=block_threads=768 TC_BATCH=12 TC_PROD_DIV=4" "BENCH_OPT=block_threads=512 TC_BATCH=16 TC_PROD_DIV=4" \
    "BENCH_OPT=block_threads=512 TC_BATCH=24 TC_PROD_DIV=4" "BENCH_OPT=block_threads=512 TC_BATCH=16" ""
  ;;
r2g)
  timeout 1200 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py > $O/r2g_pytest.txt 2>&1; echo "rc=$?" >> $O/r2g_pytest.txt
  bash scripts/gpu_ab.sh r2g C3 10 "" "TC_PROD_DIV=4" \
    "BENCH_OPT=block_threads=768 TC_BATCH=8 TC_PROD_DIV=4" "BENCH_OPT=block_threads=768 TC_BATCH=12 TC_PROD_DIV=4" \
    "BENCH_OPT=block_threads=768 TC_BATCH=16 TC_PROD_DIV=4" "BENCH_OPT=block_threads=768 TC_BATCH=12 TC_PROD_DIV=3" ""
  for c in C2 C5 C1; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2g_bench_$(echo $c | tr C c).json > $O/r2g_bench_$c.log 2>&1; done
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2g_bench_c3.json > $O/r2g_bench_c3.log 2>&1
  ;;
r2h)
  bash scripts/gpu_ab.sh r2h C3 10 "" "TC_PROD_DIV=4" "TC_PROD_DIV=3" "TC_PROD_DIV=4 TC_SLOTS=4" "TC_PROD_DIV=4 TC_SLOTS=2" "TC_PROD_DIV=4" ""
  bash scripts/gpu_ab.sh r2hc4 C4 3 "" "TC_PROD_DIV=4" "TC_PROD_DIV=3"
  ;;
r2i)
  bash scripts/gpu_ab.sh r2i C3 10 "" "TC_HEAD_PERMILLE=50 TC_HEAD_PROD_DIV=2" "TC_HEAD_PERMILLE=80 TC_HEAD_PROD_DIV=2" \
    "TC_HEAD_PERMILLE=80 TC_HEAD_PROD_DIV=3" "TC_HEAD_PERMILLE=120 TC_HEAD_PROD_DIV=3" "TC_HEAD_PERMILLE=40 TC_HEAD_PROD_DIV=2" ""
  bash scripts/gpu_ab.sh r2ic4 C4 3 "" "TC_HEAD_PERMILLE=80 TC_HEAD_PROD_DIV=2" "TC_HEAD_PERMILLE=80 TC_HEAD_PROD_DIV=3"
  ;;
r2k)
  for kv in "TC_PROD_GROUPS=2" "TC_PIPE=1"; do
    env $kv timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or partition" > $O/r2k_pytest_$(echo $kv | tr '=' '_').txt 2>&1; echo "rc=$?" >> $O/r2k_pytest_$(echo $kv | tr '=' '_').txt
  done
  bash scripts/gpu_ab.sh r2k C3 10 "" "TC_PROD_GROUPS=2" "TC_PIPE=1" "TC_PROD_GROUPS=2 TC_PIPE=1" "TC_PROD_GROUPS=2 TC_PROD_DIV=3" "TC_PROD_GROUPS=2 TC_PROD_DIV=5" ""
  bash scripts/gpu_ab.sh r2kc4 C4 3 "" "TC_PROD_GROUPS=2" "TC_PIPE=1"
  timeout 900 python -m pytest -q tests/test_gpu_balance.py -s > $O/r2k_balance1.txt 2>&1
  timeout 900 python -m pytest -q tests/test_gpu_balance.py -s > $O/r2k_balance2.txt 2>&1
  timeout 600 python bench.py --config C5 --steps 10 --warmup 3 --no-cpu-baseline --out $O/r2k_c5_bal.json > /dev/null 2>&1
  timeout 600 python bench.py --config C5 --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2k_c5_nobal.json > /dev/null 2>&1
  ;;
r2l)
  timeout 1200 python scripts/diag_refine.py --config C4 --P 8 --slices 64,128,256 > $O/r2l_refine_c4.txt 2>&1
  timeout 900 python scripts/diag_refine.py --config C3 --P 8 --slices 64,256 > $O/r2l_refine_c3.txt 2>&1
  bash scripts/gpu_ab.sh r2l C3 10 "" "TC_PROD_GROUPS=3 TC_PROD_DIV=3" "TC_PROD_GROUPS=2 TC_SLOTS=4" "TC_PROD_GROUPS=3 TC_PROD_DIV=3 TC_SLOTS=4" ""
  timeout 600 python bench.py --config C5 --steps 10 --warmup 3 --no-cpu-baseline --out $O/r2l_c5.json > /dev/null 2>&1
  ;;
r2m)
  timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py tests/test_gpu_balance.py -s > $O/r2m_pytest.txt 2>&1; echo "rc=$?" >> $O/r2m_pytest.txt
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --out $O/r2m_bench_c3.json > $O/r2m_bench_c3.log 2>&1
  TC_A5=sort timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2m_bench_c3_a5sort.json > $O/r2m_bench_c3_a5sort.log 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r2m_launches_c3.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded --no-balance > /dev/null 2>&1
  ;;
r2n)
  timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py -k "a5_paths or csr_exact or host_pipelined or full_size or closed_forms or more_than" > $O/r2n_pytest.txt 2>&1; echo "rc=$?" >> $O/r2n_pytest.txt
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2n_bench_c3.json > $O/r2n_bench_c3.log 2>&1
  TC_A5=sort timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2n_bench_c3_a5sort.json > $O/r2n_bench_c3_a5sort.log 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r2n_launches_c3.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded --no-balance > /dev/null 2>&1
  ;;
r2o)
  timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py -k "more_than" -s > $O/r2o_pytest_bigm.txt 2>&1; echo "rc=$?" >> $O/r2o_pytest_bigm.txt
  timeout 1800 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py tests/test_gpu_support.py > $O/r2o_pytest.txt 2>&1; echo "rc=$?" >> $O/r2o_pytest.txt
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-balance --out $O/r2o_bench_c3.json > $O/r2o_bench_c3.log 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r2o_launches_c3.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded --no-balance > /dev/null 2>&1
  ;;
r2p)
  bash scripts/gpu_ab.sh r2p C3 10 "" "BENCH_OPT=bitmap_factor=8" "BENCH_OPT=bitmap_factor=20" "BENCH_OPT=table_factor=4" "BENCH_OPT=table_factor=8" \
    "BENCH_OPT=chunk_cost=12288" "BENCH_OPT=chunk_cost=24576" "BENCH_OPT=seg_cost=2" "BENCH_OPT=seg_cost=8" ""
  bash scripts/gpu_ab.sh r2pc2 C2 20 "" "BENCH_OPT=table_factor=4" "BENCH_OPT=table_factor=8" "BENCH_OPT=chunk_cost=8192" "BENCH_OPT=chunk_cost=24576" ""
  ;;
r2q)
  TC_OVERLAP=1 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or partition or full_size" > $O/r2q_pytest_overlap.txt 2>&1; echo "rc=$?" >> $O/r2q_pytest_overlap.txt
  bash scripts/gpu_ab.sh r2q C3 10 "" "TC_OVERLAP=1" "BENCH_OPT=bitmap_factor=16" "BENCH_OPT=bitmap_factor=24" "BENCH_OPT=bitmap_factor=32" "TC_OVERLAP=1 BENCH_OPT=bitmap_factor=24" ""
  bash scripts/gpu_ab.sh r2qc4 C4 3 "" "TC_OVERLAP=1" "BENCH_OPT=bitmap_factor=24"
  bash scripts/gpu_ab.sh r2qc2 C2 20 "" "TC_OVERLAP=1"
  ;;
r2r)
  timeout 1800 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_support.py tests/test_gpu_fused.py > $O/r2r_pytest.txt 2>&1; echo "rc=$?" >> $O/r2r_pytest.txt
  bash scripts/gpu_ab.sh r2rc2 C2 20 "" "BENCH_OPT=bitmap_factor=12"
  bash scripts/gpu_ab.sh r2rc5 C5 20 "" "BENCH_OPT=bitmap_factor=12"
  bash scripts/gpu_ab.sh r2rc1 C1 20 "" "BENCH_OPT=bitmap_factor=12"
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --out $O/r2r_bench_c3.json > $O/r2r_bench_c3.log 2>&1
  ;;
r2s)
  timeout 600 python scripts/diag_e2e.py C3 12 > $O/r2s_e2e_c3.txt 2>&1
  TC_H2D_PIECES=4 timeout 600 python scripts/diag_e2e.py C3 6 > $O/r2s_e2e_c3_p4.txt 2>&1
  ;;
r2t)
  TC_HOSTTIME=1 timeout 600 python scripts/diag_e2e.py C3 10 > $O/r2t_e2e_c3.txt 2>&1
  ;;
r2u)
  bash scripts/gpu_abbuild.sh r2uc2 C2 20 "" "-DTC_UNROLL_SHORT=3" "-DTC_UNROLL_SHORT=4" ""
  bash scripts/gpu_abbuild.sh r2uc3 C3 10 "" "-DTC_UNROLL_SHORT=3" "-DTC_UNROLL_SHORT=4"
  bash scripts/gpu_abbuild.sh r2uc5 C5 20 "" "-DTC_UNROLL_SHORT=3" "-DTC_UNROLL_SHORT=4"
  ;;
r2v)
  bash scripts/gpu_abbuild.sh r2vc3 C3 10 "" "-DTC_L2PF=1" "" "-DTC_L2PF=1"
  bash scripts/gpu_abbuild.sh r2vc4 C4 3 "" "-DTC_L2PF=1"
  ;;
r2w)
  # The N > 1 bench path (agreed profile, ranges, sharded build, e2e, all_reduce) with
  # 2 and 4 gloo ranks sharing cuda:0 -- a test of the code path, not a scaling number.
  for N in 2 4; do
    timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 \
      --master-port 2951$N bench.py --gpus $N --steps 3 --warmup 3 --config C2 --backend gloo --share-gpu \
      --out $O/r2w_bench_c2_n$N.json > $O/r2w_bench_c2_n$N.log 2>&1; echo "rc=$?" >> $O/r2w_bench_c2_n$N.log
  done
  timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29520 bench.py --gpus 2 --steps 3 --warmup 3 --e2e-steps 1 --config C3 --backend gloo --share-gpu \
    --out $O/r2w_bench_c3_n2.json > $O/r2w_bench_c3_n2.log 2>&1; echo "rc=$?" >> $O/r2w_bench_c3_n2.log
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29530 bench.py --gpus 2 --impl reference --steps 2 --warmup 1 --config C2 \
    --out $O/r2w_reference_c2_n2.json > $O/r2w_reference_c2_n2.log 2>&1; echo "rc=$?" >> $O/r2w_reference_c2_n2.log
  ;;
r2x)
  bash scripts/gpu_abbuild.sh r2xc3 C3 10 "" "-DTC_L2PF=2" "-DTC_L2PF=3" "-DTC_PF_NEXT=1" "-DTC_L2PF=2 -DTC_PF_NEXT=1" ""
  bash scripts/gpu_abbuild.sh r2xc4 C4 3 "" "-DTC_L2PF=2" "-DTC_PF_NEXT=1"
  ;;
r2y)
  bash scripts/gpu_abbuild.sh r2yc2 C2 20 "" "-DTC_PF_SHORT=1" ""
  bash scripts/gpu_abbuild.sh r2yc3 C3 10 "" "-DTC_PF_SHORT=1"
  bash scripts/gpu_abbuild.sh r2yc5 C5 20 "" "-DTC_PF_SHORT=1"
  ;;
r2z)
  bash scripts/gpu_abbuild.sh r2zc3 C3 10 "" "-DTC_PF_ROWS=1" "-DTC_PF_FIRST=1" "-DTC_PF_ROWS=1 -DTC_PF_FIRST=1" ""
  bash scripts/gpu_abbuild.sh r2zc4 C4 3 "" "-DTC_PF_ROWS=1" "-DTC_PF_FIRST=1"
  bash scripts/gpu_abbuild.sh r2zc2 C2 20 "" "-DTC_PF_ROWS=1"
  ;;
r3a)
  BENCH_ARGS="--mode support" bash scripts/gpu_abbuild.sh r3ac3 C3 5 "" "-DTC_SUP_L2PF=1" ""
  BENCH_ARGS="--mode support" bash scripts/gpu_abbuild.sh r3ac2 C2 10 "" "-DTC_SUP_L2PF=1"
  ;;
r3b)
  bash scripts/gpu_ab.sh r3b C3 10 "" "TC_PROD_DIV=3" "TC_PROD_DIV=5" "TC_PROD_DIV=3 TC_PROD_GROUPS=3" "TC_SLOTS=4" "TC_SLOTS=2" ""
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 2 \
    -o $O/r3b_c3_count python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/r3b_ncu.log 2>&1
  python -c "import bench; print(bench.src_hash())" > $O/r3b_src_hash.txt
  ;;
r4b)
  # short class on the warp-specialised kernel (TC_SHORT_WS) vs k_count_flat
  TC_SHORT_WS=1 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or c2_chung or c5_lattice or chung_lu_small or partition or ranges or huge or cap" > $O/r4b_pytest_short_ws.txt 2>&1; echo "rc=$?" >> $O/r4b_pytest_short_ws.txt
  for c in C2 C5 C3; do
    bash scripts/gpu_ab.sh r4b_$c $c 10 "" "TC_SHORT_WS=1" "TC_SHORT_WS=1 TC_PROD_DIV_SHORT=3" "TC_SHORT_WS=1 TC_PROD_DIV_SHORT=4" "TC_SHORT_WS=1 TC_PROD_DIV_SHORT=2 TC_PROD_GROUPS=3" ""
  done
  ;;
r4c)
  # flat-kernel shape and next-chunk plan prefetch (compile-time); packed 16-B trim record in the build
  timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "csr_exact or host or dedup or options or c2_chung or c5_lattice or full_size" > $O/r4c_pytest.txt 2>&1; echo "rc=$?" >> $O/r4c_pytest.txt
  timeout 600 python bench.py --steps 10 --warmup 3 --no-sharded --no-balance --out $O/r4c_bench_c3.json > $O/r4c_bench_c3.log 2>&1
  for c in C2 C5 C3; do
    bash scripts/gpu_abbuild.sh r4c_$c $c 10 "" "-DTC_FLAT_PF=1" "-DTC_FLAT_BLOCK=256 -DTC_FLAT_CTAS=6" "-DTC_FLAT_BLOCK=192 -DTC_FLAT_CTAS=8" "-DTC_FLAT_BLOCK=512 -DTC_FLAT_CTAS=3" "-DTC_FLAT_PF=1 -DTC_FLAT_BLOCK=256 -DTC_FLAT_CTAS=6" ""
  done
  ;;
r4d)
  # tc_sort.cu radix sort vs CUB onesweep: microbenchmark, parity, build / e2e A/B at C3
  timeout 600 build/sort_bench > $O/r4d_sort_bench.txt 2>&1; echo "rc=$?" >> $O/r4d_sort_bench.txt
  timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py > $O/r4d_pytest.txt 2>&1; echo "rc=$?" >> $O/r4d_pytest.txt
  i=0; for kv in "" "TC_SORT=cub" ""; do
    i=$((i+1)); tag=${i}_$(echo "${kv:-own}" | tr ' =' '__')
    env $kv timeout 900 python bench.py --steps 10 --warmup 3 --no-balance --out $O/r4d_bench_c3_$tag.json > $O/r4d_bench_c3_$tag.log 2>&1
  done
  ;;
r4e)
  # CUB onesweep policy for the build's 64-bit key sorts (256 x 22 keys per thread) vs CUB's default
  timeout 600 build/sort_bench > $O/r4e_sort_bench.txt 2>&1; echo "rc=$?" >> $O/r4e_sort_bench.txt
  timeout 1500 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_sharded.py > $O/r4e_pytest.txt 2>&1; echo "rc=$?" >> $O/r4e_pytest.txt
  i=0; for kv in "" "TC_SORT=cub" "" "TC_SORT=cub"; do
    i=$((i+1)); tag=${i}_$(echo "${kv:-tuned}" | tr ' =' '__')
    env $kv timeout 900 python bench.py --steps 10 --warmup 3 --no-balance --out $O/r4e_bench_c3_$tag.json > $O/r4e_bench_c3_$tag.log 2>&1
  done
  ;;
r4f)
  # next batch's descriptors by shuffles (TC_XSHFL 1: x, 2: x, z, zw) vs broadcast LDS.128
  for c in C3; do
    bash scripts/gpu_abbuild.sh r4f_$c $c 10 "" "-DTC_XSHFL=1" "-DTC_XSHFL=2" "" "-DTC_XSHFL=2"
  done
  rm -f build/tc_count.o paper_conf_ipps_li0ptz24_b200/libtc.so; make -s NVEXTRA=-DTC_XSHFL=2 paper_conf_ipps_li0ptz24_b200/libtc.so > /dev/null 2>&1
  timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or full_size" > $O/r4f_pytest_xshfl2.txt 2>&1; echo "rc=$?" >> $O/r4f_pytest_xshfl2.txt
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_count -s 2 -c 1 \
    -o $O/r4f_c3_xshfl2 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-sharded --no-balance > $O/r4f_ncu.log 2>&1
  rm -f build/tc_count.o paper_conf_ipps_li0ptz24_b200/libtc.so; make -s paper_conf_ipps_li0ptz24_b200/libtc.so > /dev/null 2>&1
  ;;
r4g)
  # short class: L2 prefetch of each group's N+(v) at staging; 4 staging loads in flight per thread
  for c in C2 C5 C3; do
    bash scripts/gpu_abbuild.sh r4g_$c $c 10 "" "-DTC_PF_ROWS_SHORT=1" "-DTC_FLAT_PB=4" "-DTC_PF_ROWS_SHORT=1 -DTC_FLAT_PB=4" ""
  done
  ;;
r4h)
  # long class: one packed {first lane, bitmap flag, word base} descriptor word per tile (TC_PACKED)
  rm -f build/tc_count.o paper_conf_ipps_li0ptz24_b200/libtc.so; make -s NVEXTRA=-DTC_PACKED=1 paper_conf_ipps_li0ptz24_b200/libtc.so > /dev/null 2>&1
  timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or full_size or huge or cap or skewed" > $O/r4h_pytest_packed.txt 2>&1; echo "rc=$?" >> $O/r4h_pytest_packed.txt
  bash scripts/gpu_abbuild.sh r4h_C3 C3 10 "" "-DTC_PACKED=1" "" "-DTC_PACKED=1"
  bash scripts/gpu_abbuild.sh r4h_C4 C4 3 "" "-DTC_PACKED=1"
  ;;
r4u)
  # mbarrier try_wait suspend-time hint (TC_WAIT_HINT ns; 0 = a bare try_wait spin loop)
  bash scripts/gpu_ab.sh r4u_C3 C3 10 "" "TC_WAIT_HINT=100" "TC_WAIT_HINT=500" "TC_WAIT_HINT=2000" "TC_WAIT_HINT=10000" ""
  bash scripts/gpu_ab.sh r4u_C2 C2 10 "" "TC_WAIT_HINT=500" "TC_WAIT_HINT=2000"
  bash scripts/gpu_ab.sh r4u_C4 C4 3 "" "TC_WAIT_HINT=500" "TC_WAIT_HINT=2000"
  ;;
r4v)
  # producers' row loads in flight per lane in the insert walk (TC_INS_UNROLL, compile time)
  bash scripts/gpu_abbuild.sh r4v_C3 C3 10 "" "-DTC_INS_UNROLL=8" "-DTC_INS_UNROLL=16" ""
  bash scripts/gpu_abbuild.sh r4v_C2 C2 10 "" "-DTC_INS_UNROLL=8" "-DTC_INS_UNROLL=16"
  ;;
r4w)
  # long class only for edges whose head gets a bitmap table (TC_LONG_BITMAP): the hash-table heads of
  # the producer-bound head of the long class go to the flattened kernel
  TC_LONG_BITMAP=1 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or full_size or huge or cap or skewed or c2_chung or c5_lattice" > $O/r4w_pytest_long_bitmap.txt 2>&1; echo "rc=$?" >> $O/r4w_pytest_long_bitmap.txt
  bash scripts/gpu_ab.sh r4w_C3 C3 10 "" "TC_LONG_BITMAP=1" "" "TC_LONG_BITMAP=1"
  bash scripts/gpu_ab.sh r4w_C2 C2 10 "" "TC_LONG_BITMAP=1"
  bash scripts/gpu_ab.sh r4w_C4 C4 3 "" "TC_LONG_BITMAP=1"
  ;;
r4x)
  # hash-table heads with d+(v) <= D flattened with the short class (TC_LONG_HASH_DMAX)
  bash scripts/gpu_ab.sh r4x_C3 C3 10 "" "TC_LONG_HASH_DMAX=16" "TC_LONG_HASH_DMAX=32" "TC_LONG_HASH_DMAX=64" "TC_LONG_HASH_DMAX=128" ""
  bash scripts/gpu_ab.sh r4x_C4 C4 3 "" "TC_LONG_HASH_DMAX=32" "TC_LONG_HASH_DMAX=64"
  ;;
r4y)
  # hash table size (table_factor slots per N+(v) entry; default 6)
  bash scripts/gpu_ab.sh r4y_C3 C3 10 "" "BENCH_OPT=table_factor=3" "BENCH_OPT=table_factor=4" "BENCH_OPT=table_factor=8" ""
  bash scripts/gpu_ab.sh r4y_C2 C2 10 "" "BENCH_OPT=table_factor=3" "BENCH_OPT=table_factor=4"
  bash scripts/gpu_ab.sh r4y_C3d C3 10 "" "TC_LONG_HASH_DMAX=128" "TC_LONG_HASH_DMAX=256" "TC_LONG_HASH_DMAX=512" "TC_LONG_HASH_DMAX=1024" ""
  ;;
r5a)
  # long-class chunks taken alternately from both ends of the range by every CTA (TC_CHUNK_ORDER=1)
  TC_CHUNK_ORDER=1 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or full_size or huge or cap or skewed or partition or ranges or async" > $O/r5a_pytest_chunk_order.txt 2>&1; echo "rc=$?" >> $O/r5a_pytest_chunk_order.txt
  bash scripts/gpu_ab.sh r5a_C3 C3 10 "" "TC_CHUNK_ORDER=1" "" "TC_CHUNK_ORDER=1"
  bash scripts/gpu_ab.sh r5a_C4 C4 3 "" "TC_CHUNK_ORDER=1" "TC_LONG_HASH_DMAX=128"
  bash scripts/gpu_ab.sh r5a_C2 C2 10 "" "TC_LONG_HASH_DMAX=128" "TC_CHUNK_ORDER=1"
  bash scripts/gpu_ab.sh r5a_C3b C3 10 "TC_LONG_HASH_DMAX=128" "TC_LONG_HASH_DMAX=128 TC_CHUNK_ORDER=1" ""
  ;;
r5c)
  # e2e step spread: pool internal reuse dependencies and tc_free's device sync (A/B knobs)
  for c in C5 C3; do
    for kv in "" "TC_POOL_INTERNAL_DEPS=1" "TC_FREE_DEVSYNC=1" "TC_POOL_INTERNAL_DEPS=1 TC_FREE_DEVSYNC=1" ""; do
      tag=$(echo "${kv:-default}" | tr ' =' '__')
      env $kv timeout 900 python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 20 --no-balance --no-sharded --no-cpu-baseline --no-e2e-pipelined --out $O/r5c_${c}_$tag.json > $O/r5c_${c}_$tag.log 2>&1
      python -c "import json,sys; d=json.load(open('$O/r5c_${c}_$tag.json')); e=d['e2e']['step_ms']; print('$c', '$tag', round(sum(e)/len(e),1), [round(x) for x in e])" >> $O/r5c_e2e.txt 2>&1
    done
  done
  ;;
r5d)
  # e2e steps and the pipelined leg with pool reuse dependencies on + per-thread count result
  timeout 600 python scripts/diag_pipeline3.py > $O/r5d_pipe3.txt 2>&1
  for c in C5 C3 C2; do
    for rep in 1 2; do
      timeout 900 python bench.py --config $c --steps 3 --warmup 3 --e2e-steps 20 --no-balance --no-sharded --no-cpu-baseline --out $O/r5d_${c}_$rep.json > $O/r5d_${c}_$rep.log 2>&1
      python -c "import json; d=json.load(open('$O/r5d_${c}_$rep.json')); e=d['e2e']['step_ms']; print('$c', $rep, round(sum(e)/len(e),1), [round(x) for x in e], 'pipelined', round(d['e2e_pipelined']['ms_per_step'],1))" >> $O/r5d_e2e.txt 2>&1
    done
  done
  ;;
r5i)
  # consumers insert N+(v) of insert-heavy long-class chunks (TC_CONS_INSERT = R: when inserts x R > key lanes)
  TC_CONS_INSERT=1 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py -k "closed_forms or c1_rmat10 or rmat_medium or options or karate or golden or full_size or huge or cap or skewed or partition or ranges" > $O/r5i_pytest_cons_insert.txt 2>&1; echo "rc=$?" >> $O/r5i_pytest_cons_insert.txt
  TC_CONS_INSERT=1000 TC_CUCKOO_KICKS=0 timeout 900 python -m pytest -q -x tests/test_gpu_parity.py tests/test_gpu_robust.py -k "closed_forms or c1_rmat10 or rmat_medium or options or cuckoo" > $O/r5i_pytest_cons_insert_cuckoo.txt 2>&1; echo "rc=$?" >> $O/r5i_pytest_cons_insert_cuckoo.txt
  bash scripts/gpu_ab.sh r5i_C3 C3 10 "" "TC_CONS_INSERT=1" "TC_CONS_INSERT=2" "TC_CONS_INSERT=4" "TC_CONS_INSERT=16" ""
  bash scripts/gpu_ab.sh r5i_C4 C4 3 "" "TC_CONS_INSERT=2" "TC_CONS_INSERT=4"
  ;;
r6b)
  # chunk sizes (plan option chunk_cost: long chunks 4x, short 1x) and the short-class divisor
  bash scripts/gpu_ab.sh r6b_C3 C3 10 "" "BENCH_OPT=chunk_cost=12288" "BENCH_OPT=chunk_cost=24576" "BENCH_OPT=chunk_cost=32768" "TC_CS_DIV=2" ""
  bash scripts/gpu_ab.sh r6b_C2 C2 10 "" "BENCH_OPT=chunk_cost=12288" "BENCH_OPT=chunk_cost=24576" "BENCH_OPT=chunk_cost=32768" "TC_CS_DIV=2"
  bash scripts/gpu_ab.sh r6b_C5 C5 10 "" "BENCH_OPT=chunk_cost=8192" "BENCH_OPT=chunk_cost=24576"
  ;;
r6c)
  # flat kernel: 3 CTAs x 384 threads (54 registers) with 3 / 4 tiles of keys in flight per warp
  for c in C2 C5 C3; do
    bash scripts/gpu_abbuild.sh r6c_$c $c 10 "" "-DTC_FLAT_CTAS=3 -DTC_UNROLL_SHORT=3" "-DTC_FLAT_CTAS=3 -DTC_UNROLL_SHORT=4" ""
  done
  ;;
r6d)
  # long-class chunk cost multiplier (TC_LONG_CHUNK; long chunks = x * chunk_cost, default 4)
  bash scripts/gpu_ab.sh r6d_C3 C3 10 "" "TC_LONG_CHUNK=5" "TC_LONG_CHUNK=6" "TC_LONG_CHUNK=8" "TC_LONG_CHUNK=12" ""
  bash scripts/gpu_ab.sh r6d_C2 C2 10 "" "TC_LONG_CHUNK=6" "TC_LONG_CHUNK=8"
  bash scripts/gpu_ab.sh r6d_C4 C4 3 "" "TC_LONG_CHUNK=6" "TC_LONG_CHUNK=8"
  ;;
*) echo "unknown tag $T"; exit 1;;
esac
echo done > $O/${T}_done.txt
