set -x
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_long_query_gpu.py tests/test_f2_workloads_gpu.py -q -p no:cacheprovider -x -k "gangs or long_sequence or auto or long_query or forced or protein or alphabet or recompute or tmode or variance or table2" 2>&1 | tail -3 > gpurun_out/r02q_tests.txt
for m in 144 567 1500; do timeout 120 python tools/profile_long.py $m 3073 3 C3 | tail -1; done > gpurun_out/r02q_perf.txt 2>&1
for T in 3072 2572 1172 512 0; do timeout 120 python tools/profile_long.py 567 $T 3 C2 | tail -1; done >> gpurun_out/r02q_perf.txt 2>&1
