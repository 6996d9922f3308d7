set -x
ncu --set full --clock-control none --import-source on -k regex:k_search_t -s 2 -c 1 -o gpurun_out/r02c_tlong_c2 -f python tools/profile_long.py 567 3072 3 C2 > gpurun_out/r02c_tlong_c2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_search_t -s 2 -c 1 -o gpurun_out/r02c_tlong_c3 -f python tools/profile_long.py 567 3073 3 C3 > gpurun_out/r02c_tlong_c3.log 2>&1
for e in "" "SW_T_GANG=0:0" "SW_T_TEAM=4" "SW_T_TEAM=2" "SW_T_GANG=8" "SW_T_GANG=2"; do python tools/profile_long.py 567 3072 3 C2 "$e" | tail -1 | sed "s/^/[$e] /"; done > gpurun_out/r02c_variants.txt 2>&1
