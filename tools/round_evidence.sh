# Round evidence in one gpurun call (one GPU): GPU parity tests, smoke, bench line (ours and
# the oracle reference arm), C4 / C5 lines under torchrun (world 1, NCCL path on), the ncu
# launch list of a bench run, one `ncu --set full` capture of the top kernel (query 5478 on C2,
# -> profiles/traffic.json) and of the T-mode kernel, and the sweeps.
#   bash tools/round_evidence.sh TAG [quick]
TAG=${1:-ev}
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > $O/gpu.txt 2>&1
lscpu > $O/lscpu.txt 2>&1
timeout 600 python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -20 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; tail -3 $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench.jsonl 2> $O/bench.err; tail -c 600 $O/bench.jsonl
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.jsonl 2> $O/bench_ref.err; tail -c 300 $O/bench_ref.jsonl
SW_BENCH_DIST=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 \
    --master-port 29517 bench.py --gpus 1 --config C4 --steps 5 --warmup 3 > $O/bench_c4_torchrun.jsonl 2> $O/bench_c4_torchrun.err
C5_SHARDS=8 SW_BENCH_DIST=1 timeout 1500 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 \
    --master-addr 127.0.0.1 --master-port 29518 bench.py --gpus 1 --config C5 --steps 1 --warmup 3 --no-auto --no-stream \
    --cpu-budget 8 > $O/bench_c5_torchrun.jsonl 2> $O/bench_c5_torchrun.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-auto --no-stream > $O/ncu_bench.log 2>&1
python tools/summarize_launches.py $O/launches.csv > $O/launches_summary.txt 2>&1; head -12 $O/launches_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled \
    -k regex:8k_searchINS_9LaneS16x2 -c 1 -o $O/full_m5478 -f python tools/profile_one.py 5478 3072 1 > $O/full_m5478.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_search_t -s 2 -c 1 -o $O/full_tmode_c3_567 -f \
    python tools/profile_long.py 567 3073 3 C3 > $O/full_tmode.log 2>&1
[ "$2" = "quick" ] && exit 0
Ts=$(python -c "print(','.join(str(t) for t in list(range(3072,1171,-100))+[1024,512,0,36000]))")
timeout 1500 python tools/sweep_threshold.py C2 567 $Ts > $O/sweep_c2_567.jsonl 2> $O/sweep_c2_567.err
for m in 144 375 729 1500 5478; do timeout 600 python tools/sweep_threshold.py C3 $m 36000,16384,8192,6144,4096,3073,auto; done > $O/sweep_c3.jsonl 2> $O/sweep_c3.err
timeout 900 python tools/variance_sweep.py > $O/variance.jsonl 2> $O/variance.err
timeout 1500 python tools/table2_sweep.py > $O/table2.jsonl 2> $O/table2.err
timeout 900 python tools/query_sweep.py 3072 > $O/q20_T3072.jsonl 2>&1
timeout 900 python tools/query_sweep.py -1 > $O/q20_auto.jsonl 2>&1
ls -la $O
