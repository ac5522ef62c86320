# one ncu --set full capture of the long-class count kernel at config C3 (+ the short-class one)
TAG=${1:-r18b}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_count$" -s 1 -c 1 -o gpurun_out/${TAG}_prof_c3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/${TAG}_ncu_log.txt 2>&1
