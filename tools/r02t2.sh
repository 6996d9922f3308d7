mkdir -p gpurun_out/t3
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/t3/pytest.log 2>&1; tail -3 gpurun_out/t3/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
Ts=$(python -c "print(','.join(str(t) for t in [3072,2572,2072,1572,1172,512,0,36000]))")
timeout 900 python tools/sweep_threshold.py C2 144 $Ts > gpurun_out/t3/sweep_c2_144.jsonl 2> gpurun_out/t3/sweep_c2_144.err
python - <<'P'
import json
for l in open('gpurun_out/t3/sweep_c2_144.jsonl'):
    d=json.loads(l); print(d['T'], d['gcups_total'], d.get('gcups_long_only'), d.get('gcups_short_only'), d.get('long_over_short'))
P
