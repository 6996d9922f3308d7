timeout 900 python tools/query_sweep.py 3072 > gpurun_out/q20_1.jsonl 2>&1; cat gpurun_out/q20_1.jsonl | python -c "
import sys,json
for l in sys.stdin:
  try: d=json.loads(l); print(d['m'], d['gcups'], end='; ')
  except: pass
"; echo
timeout 900 python tools/query_sweep.py 3072 > gpurun_out/q20_2.jsonl 2>&1; cat gpurun_out/q20_2.jsonl | python -c "
import sys,json
for l in sys.stdin:
  try: d=json.loads(l); print(d['m'], d['gcups'], end='; ')
  except: pass
"; echo
