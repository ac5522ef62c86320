# ncu --set full of k_count + k_count_flat at C3 and k_count_flat at C2, plus the C3 launch list
TAG=${1:-r19h}
O=gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_count$" -s 1 -c 1 -o $O/${TAG}_prof_c3 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded > $O/${TAG}_ncu_log.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_count_flat" -s 1 -c 1 -o $O/${TAG}_prof_c3_flat python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded >> $O/${TAG}_ncu_log.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_count_flat" -s 1 -c 1 -o $O/${TAG}_prof_c2_flat python bench.py --config C2 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded >> $O/${TAG}_ncu_log.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/${TAG}_launches_c3.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-sharded > /dev/null 2>&1
echo done > $O/${TAG}_done.txt
