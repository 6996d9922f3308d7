for v in 0 1 0 1; do SW_STREAM_TUNED=$v timeout 900 python bench.py --no-cpu-baseline --no-auto > gpurun_out/st$v.jsonl 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/st$v.jsonl').read().strip().splitlines()[-1]); print('tuned=$v', d['value'], d['stream_db']['value'], d['stream_db']['seconds'])"; done
