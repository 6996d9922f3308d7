"""Drive one search of the C2 database with a single query (for ncu / nsys-style captures).
usage: python tools/profile_one.py [query_len=5478] [threshold=3072] [reps=2] [config=C2]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

L = int(sys.argv[1]) if len(sys.argv) > 1 else 5478
T = int(sys.argv[2]) if len(sys.argv) > 2 else 3072
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
cfg = sys.argv[4] if len(sys.argv) > 4 else "C2"
q = gen.make_query(L)
if os.environ.get("SW_LIB"):          # A/B against another build of the library
    swp.load_library(os.environ["SW_LIB"])
if cfg == "C3":
    lens = gen.long_lengths(4096, seed=3)
    db = gen.build_database(lens, 3, [q])
else:
    lens = gen.sp_lengths(540_000, seed=2)
    db = gen.build_database(lens, 2, [q])
with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    for _ in range(reps):
        t0 = time.perf_counter()
        out = sw.search(T)
        dt = time.perf_counter() - t0
        km = sw.kernel_ms()
        cells = L * db.total_residues
        print(f"m={L} T={T} wall={dt*1e3:.1f} ms kernel={km['search_ms']:.2f} ms "
              f"recompute={km['recompute_ms']:.3f} ms -> {cells / (km['search_ms'] / 1e3) / 1e9:.1f} GCUPS (kernel)",
              flush=True)
