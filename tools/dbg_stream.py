"""Debug helper: streamed search per query on the C2 database (usage: python tools/dbg_stream.py [chunk])."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

chunk = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 25
n = int(sys.argv[2]) if len(sys.argv) > 2 else 540_000
lens = gen.sp_lengths(n, seed=2)
db = gen.build_database(lens, 2, None)
for m in ([int(sys.argv[3])] if len(sys.argv) > 3 else gen.BENCH_QUERY_LENGTHS):
    q = gen.make_query(m)
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        ref = sw.search(3072)
        try:
            got = sw.search_stream(db.residues, db.offsets, 3072, chunk)
            print(m, "stream ok", bool(np.array_equal(got.reshape(-1), ref)), flush=True)
        except swp.SWError as e:
            print(m, "stream FAIL", e, flush=True)
            break
