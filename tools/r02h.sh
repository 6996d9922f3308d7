set -x
timeout 900 python -m pytest tests/test_parity_gpu.py -q -p no:cacheprovider -x -k "gangs or long_sequence" 2>&1 | tail -5 > gpurun_out/r02h_tests.txt
for e in "SW_T_GANG_CHAIN2=0" "SW_T_GANG_CHAIN2=1"; do
  for sel in top:2 ""; do
    for T in 3072 2572; do python tools/profile_long.py 567 $T 3 C2 "$e" "$sel" | tail -1 | sed "s/^/[$e $sel] /"; done
  done
done > gpurun_out/r02h_var.txt 2>&1
for g in 4:1 6:1 8:1; do python tools/profile_long.py 567 3072 3 C2 "SW_T_GANG=$g" top:2 | tail -1 | sed "s/^/[gang $g top:2] /"; done >> gpurun_out/r02h_var.txt 2>&1
