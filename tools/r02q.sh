timeout 900 python tools/query_sweep.py 3072 > gpurun_out/q20_T3072.jsonl 2>&1; cat gpurun_out/q20_T3072.jsonl | python -c "
import sys,json
for l in sys.stdin:
  try: d=json.loads(l); print(d['m'], d['gcups'], end='; ')
  except: pass
"
timeout 900 python -m pytest tests/test_parity_gpu.py -q -p no:cacheprovider -k "every_config" 2>&1 | tail -1
