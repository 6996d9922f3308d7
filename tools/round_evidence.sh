# Round evidence in one gpurun call (one GPU): GPU parity tests, smoke, bench line (ours and
# the oracle reference arm), the ncu launch list of a bench run and one `ncu --set full`
# capture of the top kernel (query 5478 on C2).
#   bash tools/round_evidence.sh TAG
TAG=${1:-ev}
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -20 $O/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1; tail -3 $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench.jsonl 2> $O/bench.err; tail -c 600 $O/bench.jsonl
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.jsonl 2> $O/bench_ref.err; tail -c 300 $O/bench_ref.jsonl
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-auto --no-stream > $O/ncu_bench.log 2>&1
python tools/summarize_launches.py $O/launches.csv > $O/launches_summary.txt 2>&1; head -12 $O/launches_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled \
    -k regex:8k_searchINS_9LaneS16x2 -c 1 -o $O/full_m5478 -f python tools/profile_one.py 5478 3072 1 > $O/full_m5478.log 2>&1
ls -la $O
