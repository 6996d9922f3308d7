set -x
timeout 900 python -m pytest tests/test_parity_gpu.py -q -p no:cacheprovider -x -k "gangs or auto or long_sequence" 2>&1 | tail -5 > gpurun_out/r02d_tests.txt
for e in "SW_T_GANG_SHARE=0" "SW_T_GANG_SHARE=1" "SW_T_GANG_SHARE=1;SW_T_GANG=8" "SW_T_GANG_SHARE=1;SW_T_GANG=6:24" "SW_T_GANG_SHARE=1;SW_T_GANG=3:32"; do
  for T in 3072 2572; do python tools/profile_long.py 567 $T 3 C2 "$e" | tail -1 | sed "s/^/[$e] /"; done
done > gpurun_out/r02d_variants.txt 2>&1
SW_DEBUG_PLAN=1 python tools/sweep_threshold.py C3 144 auto,3073 > gpurun_out/r02d_c3auto.jsonl 2> gpurun_out/r02d_c3auto.err
