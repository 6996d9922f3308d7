timeout 600 python -m pytest tests/test_parity_gpu.py -q -p no:cacheprovider -x -k "gangs" 2>&1 | tail -3 > gpurun_out/r02k_tests.txt
SW_DEBUG_GANG_TIMES=1 python tools/profile_long.py 567 3072 2 C2 "SW_T_GANG=8:1" top:2 > gpurun_out/r02k_m567.txt 2>&1
for sel in top:2 ""; do for T in 3072 2572; do python tools/profile_long.py 567 $T 3 C2 "" "$sel" | tail -1 | sed "s/^/[$sel] /"; done; done > gpurun_out/r02k_var.txt 2>&1
for g in 4:1 6:1 8:1; do python tools/profile_long.py 567 3072 3 C2 "SW_T_GANG=$g" top:2 | tail -1 | sed "s/^/[gang $g top:2] /"; done >> gpurun_out/r02k_var.txt 2>&1
