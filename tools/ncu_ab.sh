# A/B ncu metrics of the main search kernel for (SW_GROUP_STREAM, SW_FORCE_MENU) pairs.
# usage: bash tools/ncu_ab.sh QUERY_LEN "stream menu" ["stream menu" ...]
L=$1; shift
M=gpu__time_duration.sum,smsp__inst_executed.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__average_warps_issue_stalled_wait_per_issue_active.ratio,smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio,smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_branch_resolving_per_issue_active.ratio,smsp__average_warps_issue_stalled_no_instruction_per_issue_active.ratio,smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio,smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio,smsp__average_warps_issue_stalled_selected_per_issue_active.ratio,smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio,smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio,smsp__thread_inst_executed_per_inst_executed.ratio,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio,smsp__average_warps_issue_stalled_membar_per_issue_active.ratio
mkdir -p gpurun_out
for cfg in "$@"; do set -- $cfg
  echo "=== stream=$1 menu=$2 m=$L"
  SW_GROUP_STREAM=$1 SW_FORCE_MENU=$2 ncu --clock-control none --kernel-name-base mangled -k regex:8k_search -c 1 \
    --metrics $M --csv --log-file gpurun_out/ncu_tmp.csv python tools/profile_one.py $L 3072 1 > /dev/null 2>&1
  python -c "
import csv
r=list(csv.reader(l for l in open('gpurun_out/ncu_tmp.csv') if not l.startswith('==')))
h=r[0]
for row in r[1:]:
    d=dict(zip(h,row)); print(d['Metric Name'].replace('smsp__average_warps_issue_stalled_','stall_').replace('_per_issue_active.ratio',''), d['Metric Value'])
"
done
