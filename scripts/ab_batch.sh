# A/B: the in-tree build, then a rebuild with NVEXTRA="$1" (e.g. -DTC_BATCH_LONG=4)
bash scripts/gpu_quick.sh
echo "NVEXTRA=$1" >> gpurun_out/quick.txt
touch paper_conf_ipps_li0ptz24_b200/csrc/tc_count.cu; make -s NVEXTRA="$1" > /dev/null 2>&1
bash scripts/gpu_quick.sh
