# copy a round_evidence.sh run (gpurun_out/TAG) into profiles/ under round-2 names
T=gpurun_out/${1:-r02ev2}; P=profiles
cp $T/bench.jsonl $P/r02_bench_latest.jsonl
cp $T/bench_ref.jsonl $P/r02_bench_reference.jsonl
cp $T/bench_c4_torchrun.jsonl $P/r02_bench_c4_world1.jsonl
cp $T/bench_c5_torchrun.jsonl $P/r02_bench_c5_shard8.jsonl
cp $T/launches.csv $P/r02_launches_bench_step.csv
cp $T/launches_summary.txt $P/r02_launches_bench_step.txt
[ -f $T/sweep_c2_567.jsonl ] && cp $T/sweep_c2_567.jsonl $P/r02_sweep_c2_567.jsonl
[ -f $T/sweep_c3.jsonl ] && cp $T/sweep_c3.jsonl $P/r02_sweep_c3_all.jsonl
[ -f $T/variance.jsonl ] && cp $T/variance.jsonl $P/r02_variance_sweep.jsonl
[ -f $T/table2.jsonl ] && cp $T/table2.jsonl $P/r02_table2_sweep.jsonl
[ -f $T/q20_T3072.jsonl ] && cp $T/q20_T3072.jsonl $P/r02_query_sweep_T3072.jsonl
[ -f $T/q20_auto.jsonl ] && cp $T/q20_auto.jsonl $P/r02_query_sweep_auto.jsonl
cp $T/lscpu.txt $P/r02_lscpu.txt
python tools/ncu_summary.py $T/full_m5478.ncu-rep "ncu --set full --clock-control none, k_search<LaneS16x2,32,43,43,384> multi-strip kernel (query 5478 on C2, T=3072), round-2 final build; tools/round_evidence.sh $1" > $P/r02_ncu_k_search_m5478_summary.txt
python tools/ncu_summary.py $T/full_tmode_c3_567.ncu-rep "ncu --set full --clock-control none, k_search_t<16,256> (T-mode, C3 all-long at T=3073, query 567), round-2 final build; tools/round_evidence.sh $1" > $P/r02_ncu_k_search_t_c3_567_summary.txt
python tools/traffic_from_ncu.py $T/full_m5478.ncu-rep
