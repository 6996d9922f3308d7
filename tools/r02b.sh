# round 2 GPU run b: new parity tests (wide penalties, long queries, updated limits), T-mode perf check
set -x
timeout 1500 python -m pytest tests/test_wide_params_gpu.py tests/test_long_query_gpu.py tests/test_parity_gpu.py -q -p no:cacheprovider -x 2>&1 | tail -30 > gpurun_out/r02b_tests.txt
timeout 600 python tools/sweep_threshold.py C3 567 3073 > gpurun_out/r02b_c3_567.jsonl 2>&1
timeout 600 python tools/sweep_threshold.py C3 144 3073 >> gpurun_out/r02b_c3_567.jsonl 2>&1
timeout 300 python tools/long_tail_probe.py 567 3072 > gpurun_out/r02b_tail.txt 2>&1
