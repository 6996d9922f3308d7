# quick A/B after a kernel change (under gpurun): GPU parity tests, C2 query sweep, C3 all-long.
#   bash tools/ab_run.sh TAG
TAG=${1:-ab}
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.log 2>&1
tail -3 gpurun_out/${TAG}_pytest.log
timeout 300 python tools/query_sweep.py 3072 144,375,729,1500,5478 > gpurun_out/${TAG}_qsweep.jsonl 2>&1
for m in 144 567 5478; do timeout 200 python tools/sweep_threshold.py C3 $m 3073; done > gpurun_out/${TAG}_c3.jsonl 2>&1
cat gpurun_out/${TAG}_qsweep.jsonl gpurun_out/${TAG}_c3.jsonl
