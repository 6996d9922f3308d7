timeout 900 python -m pytest tests -m gpu -v -p no:cacheprovider --timeout 120 --timeout-method thread -x 2>&1 | grep -E "PASS|FAIL|ERROR|Timeout|passed|failed|File .*sw_|Stack of" | tail -30 > gpurun_out/r02t_tests.txt
for m in 144 567 1500; do timeout 60 python tools/profile_long.py $m 3073 3 C3 | tail -1; done > gpurun_out/r02t_perf.txt 2>&1
for T in 3072 2572 1172 512 0; do timeout 60 python tools/profile_long.py 567 $T 3 C2 | tail -1; done >> gpurun_out/r02t_perf.txt 2>&1
