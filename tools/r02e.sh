set -x
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_long_query_gpu.py tests/test_wide_params_gpu.py tests/test_parity_full_gpu.py -q -p no:cacheprovider -x -k "gangs or auto or long_sequence or long_query or alphabet or large_pen or c3_full or protein or forced or recompute" 2>&1 | tail -5 > gpurun_out/r02e_tests.txt
for tc in 0 1; do
  for m in 144 567 1500; do python tools/profile_long.py $m 3073 3 C3 "SW_T_TWO_COL=$tc" | tail -1 | sed "s/^/[2col=$tc] /"; done
  for T in 3072 2572 1172; do python tools/profile_long.py 567 $T 3 C2 "SW_T_TWO_COL=$tc" | tail -1 | sed "s/^/[2col=$tc] /"; done
done > gpurun_out/r02e_variants.txt 2>&1
