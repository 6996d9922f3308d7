set -x
SW_DEBUG_PLAN=1 python tools/profile_long.py 567 3072 2 C2 "" top:2 > gpurun_out/r02g_plan.txt 2>&1
for g in 2:1 3:1 4:1 5:1 6:1 8:1; do
  python tools/profile_long.py 567 3072 3 C2 "SW_T_GANG=$g" top:2 | tail -1 | sed "s/^/[gang $g top:2] /"
done > gpurun_out/r02g_gang.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_search_t -s 2 -c 1 -o gpurun_out/r02g_top2 -f python tools/profile_long.py 567 3072 3 C2 "" top:2 > gpurun_out/r02g_ncu.log 2>&1
