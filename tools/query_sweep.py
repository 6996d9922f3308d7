"""GCUPS of one search per query length on the C2 database (Fig.7 analog: GCUPS vs
query length).  usage: python tools/query_sweep.py [T] [len,len,...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

T = int(sys.argv[1]) if len(sys.argv) > 1 else 3072
Ls = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else gen.BENCH_QUERY_LENGTHS
if os.environ.get("SW_LIB"):          # A/B against another build of the library
    swp.load_library(os.environ["SW_LIB"])
lens = gen.sp_lengths(540_000, seed=2)
db = gen.build_database(lens, 2, None)
with swp.SmithWaterman(gen.make_query(144), BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    for m in Ls:
        sw.set_query(gen.make_query(m))
        sw.search(T)
        ms = 1e30
        for _ in range(int(os.environ.get("SW_REPS", "1"))):
            sw.search(T)
            ms = min(ms, sw.kernel_ms()["search_ms"])
        print(json.dumps({"m": m, "T": sw.last_threshold(), "kernel_ms": round(ms, 3),
                          "gcups": round(m * db.total_residues / ms / 1e6, 1)}), flush=True)
