"""Kernel time of every menu entry for given query lengths and thresholds on the C2 database.
usage: python tools/sweep_menu.py "144,375" "3072,1073741824" "0,1,3,9" """
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

Ls = [int(x) for x in sys.argv[1].split(",")]
Ts = [int(x) for x in sys.argv[2].split(",")]
menus = [int(x) for x in sys.argv[3].split(",")]
cfg = sys.argv[4] if len(sys.argv) > 4 else "C2"
if cfg == "C3":
    lens = gen.long_lengths(4096, seed=3)
    db = gen.build_database(lens, 3, None)
else:
    lens = gen.sp_lengths(540_000, seed=2)
    db = gen.build_database(lens, 2, None)
L = db.lengths
with swp.SmithWaterman(gen.make_query(144), BLOSUM62, 10, 2) as sw:
    sw.load_db(db.residues, db.offsets)
    for m in Ls:
        q = gen.make_query(m)
        sw.set_query(q)
        for T in Ts:
            cells_long = m * int(L[L >= T].sum())
            cells = m * int(L.sum())
            for mu in menus:
                os.environ["SW_FORCE_MENU"] = str(mu)
                try:
                    sw.search(T)
                    sw.search(T)
                except swp.SWError as e:
                    print(f"m={m} T={T} menu={mu}: {e}")
                    continue
                ms = sw.kernel_ms()["search_ms"]
                print(f"m={m} T={T} menu={mu} kernel={ms:.2f} ms GCUPS={cells / ms / 1e6:.0f} "
                      f"long_cells={cells_long / cells:.3f}", flush=True)
