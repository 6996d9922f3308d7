# Threshold sweeps (Fig.3/Fig.5 analogs) on the current build (under gpurun):
#   bash tools/sweeps_all.sh TAG
TAG=${1:-sw}
mkdir -p gpurun_out
python tools/sweep_threshold.py C2 567 3072,2572,2072,1572,1172,16384,auto > gpurun_out/${TAG}_c2_567.jsonl 2>&1
for m in 144 567 1500 5478; do python tools/sweep_threshold.py C3 $m 36000,16384,8192,6144,4096,3073,auto; done > gpurun_out/${TAG}_c3.jsonl 2>&1
python tools/query_sweep.py 3072 > gpurun_out/${TAG}_q20_T3072.jsonl 2>&1
python tools/query_sweep.py -1 > gpurun_out/${TAG}_q20_auto.jsonl 2>&1
