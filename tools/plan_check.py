"""Planner check: for each query length, the kernel time of every menu entry (SW_FORCE_MENU) and of
the planner's own choice on the C2 database at T (default 3072).
usage: python tools/plan_check.py [T] [len,len,...] [menu,menu,...]  -> one JSON line per length"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from paper_conf_ipps_hainscobr11_b200 import load_library  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

T = int(sys.argv[1]) if len(sys.argv) > 1 else 3072
Ls = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 and sys.argv[2] else gen.BENCH_QUERY_LENGTHS
menus = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [i for i in range(41) if i != 11]
lens = gen.sp_lengths(540_000, seed=2)
db = gen.build_database(lens, 2, None)
with swp.SmithWaterman(gen.make_query(144), BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    for m in Ls:
        sw.set_query(gen.make_query(m))
        times = {}
        for mu in [None] + menus:
            if mu is None:
                os.environ.pop("SW_FORCE_MENU", None)
            else:
                os.environ["SW_FORCE_MENU"] = str(mu)
            try:
                sw.search(T)
                sw.search(T)
            except swp.SWError:
                continue
            times["plan" if mu is None else mu] = sw.kernel_ms()["search_ms"]
        os.environ.pop("SW_FORCE_MENU", None)
        best = min((v, k) for k, v in times.items() if k != "plan")
        print(json.dumps({"m": m, "T": T, "plan_ms": round(times["plan"], 3), "best_menu": best[1],
                          "best_ms": round(best[0], 3), "plan_over_best": round(times["plan"] / best[0], 4),
                          "all": {str(k): round(v, 3) for k, v in sorted(times.items(), key=lambda x: x[1])[:6]}}),
              flush=True)
