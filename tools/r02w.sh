mkdir -p gpurun_out/w2
timeout 900 python -m pytest tests/test_abi_gpu.py -q -p no:cacheprovider -x 2>&1 | tail -1
for i in 1 2; do timeout 900 python bench.py --no-cpu-baseline --no-stream > gpurun_out/w2/bench$i.jsonl 2> gpurun_out/w2/bench$i.err; python -c "
import json; d=json.loads(open('gpurun_out/w2/bench$i.jsonl').read().strip().splitlines()[-1]); print(d['value'], d['e2e']['value'], d['roofline']['frac'], d['parity']['mismatches'], d['auto_threshold']['value'])"; done
