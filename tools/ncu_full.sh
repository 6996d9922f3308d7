# ncu --set full captures used for the roofline analysis (run under gpurun, one GPU).
#   bash tools/ncu_full.sh TAG [QUERY_LEN ...]
# -> gpurun_out/<TAG>_cellmix.ncu-rep (the int_peaks cell-mix microbenchmark, the roofline denominator)
#    gpurun_out/<TAG>_m<L>.ncu-rep     (the main k_search launch of one C2 search with query L)
TAG=$1; shift
mkdir -p gpurun_out
ncu --set full --clock-control none -k regex:k_cellmix -c 1 -o gpurun_out/${TAG}_cellmix -f tools/int_peaks > /dev/null 2>&1
for L in "$@"; do
  ncu --set full --clock-control none --import-source on --kernel-name-base mangled \
      -k regex:8k_searchINS_9LaneS16x2 -c 1 -o gpurun_out/${TAG}_m$L -f python tools/profile_one.py $L 3072 1 > gpurun_out/${TAG}_m$L.log 2>&1
done
