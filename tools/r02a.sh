set -x
nproc; lscpu | grep "Model name"
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -40 > gpurun_out/r02a_tests.txt
timeout 600 python bench.py > gpurun_out/r02a_bench.jsonl 2> gpurun_out/r02a_bench.err
timeout 300 python tools/long_tail_probe.py 567 3072 > gpurun_out/r02a_tail.txt 2>&1
SW_DEBUG_PLAN=1 timeout 300 python tools/long_tail_probe.py 567 2572 > gpurun_out/r02a_tail2572.txt 2>&1
