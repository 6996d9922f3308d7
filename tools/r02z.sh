mkdir -p gpurun_out/t2
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/t2/pytest.log 2>&1; tail -3 gpurun_out/t2/pytest.log
SW_DEBUG_PLAN=1 timeout 300 python tools/query_sweep.py 3072 729,1500,5478 2>&1 | grep -E "tune m|gcups"
