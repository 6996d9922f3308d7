# short-path A/B (single-strip plain groups) + GPU tests + the C2 query-567 threshold sweep on the current build
bash tools/ab_short.sh abs2
Ts=$(python -c "print(','.join(str(t) for t in list(range(3072,1171,-100))+[1024,512,0,36000]))")
timeout 1500 python tools/sweep_threshold.py C2 567 $Ts > gpurun_out/abs2/sweep_c2_567.jsonl 2> gpurun_out/abs2/sweep_c2_567.err
tail -5 gpurun_out/abs2/sweep_c2_567.jsonl
