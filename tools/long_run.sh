mkdir -p gpurun_out
for m in 144 567 1500 5478; do python tools/sweep_threshold.py C3 $m 3073; done > gpurun_out/c3_long.jsonl 2>&1
python tools/sweep_threshold.py C2 567 3072,2072,1172 > gpurun_out/c2_sweep567.jsonl 2>&1
for m in 144 567; do
ncu --set full --clock-control none --import-source on -k regex:k_search_t -c 1 -o gpurun_out/tmode_m$m -f python tools/profile_one.py $m 0 1 C3 > /dev/null 2>&1
done
