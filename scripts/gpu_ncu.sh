# ncu --set full of one launch of each count kernel per config.
# usage: bash scripts/gpu_ncu.sh TAG C3 [C2 ...]   (K=k_count|k_count_flat|both, default both)
TAG=$1; shift
make -j8 >/dev/null 2>&1 || make
mkdir -p gpurun_out
for c in "$@"; do
  lc=$(echo $c | tr 'A-Z' 'a-z')
  for k in ${K:-k_count k_count_flat}; do
    suffix=$([ "$k" = "k_count" ] && echo "" || echo "_flat")
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:"^${k}\$" -s 1 -c 1 -o gpurun_out/${TAG}_prof_${lc}${suffix} python bench.py --config $c --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/${TAG}_ncu_${lc}${suffix}.log 2>&1
    tail -1 gpurun_out/${TAG}_ncu_${lc}${suffix}.log
  done
done
