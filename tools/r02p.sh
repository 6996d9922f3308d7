set -x
for n in 20000 100000; do
timeout 60 python - <<PY 2>&1 | tail -2
import os, sys, time
sys.path.insert(0, '.')
import numpy as np
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM62
lens = gen.sp_lengths($n, seed=2)
db = gen.build_database(lens, 2, None)
q = gen.make_query(567)
with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    for T in (0, 0, 512):
        t0 = time.time(); sw.search(T); print('n=$n T', T, 'ok', time.time() - t0, sw.kernel_ms(), flush=True)
PY
done > gpurun_out/r02p_small.txt 2>&1
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_long_query_gpu.py -q -p no:cacheprovider -x -k "gangs or long_sequence or auto or long_query or forced or protein or alphabet or recompute or tmode" 2>&1 | tail -3 > gpurun_out/r02p_tests.txt
for T in 3072 2572 1172 512 0; do timeout 120 python tools/profile_long.py 567 $T 3 C2 | tail -1; done > gpurun_out/r02p_perf.txt 2>&1
