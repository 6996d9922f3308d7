set -x
for n in 2000 20000 100000; do
timeout 90 python - <<PY 2>&1 | tail -8
import os, sys, time
sys.path.insert(0, '.')
os.environ['SW_DEBUG_PLAN'] = '1'
import numpy as np
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM62
lens = gen.sp_lengths($n, seed=2)
db = gen.build_database(lens, 2, None)
q = gen.make_query(567)
with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    t0 = time.time(); sw.search(0); print('n=$n T=0 search ok', time.time() - t0, sw.kernel_ms(), flush=True)
PY
done
