"""Engine probe on idealised databases: N sequences of one fixed length (no length variance, no
long path), one query, a forced menu entry; kernel GCUPS and cells/clk/GPU.
usage: python tools/uniform_probe.py m menu len1,len2,... [n_residues=2e8]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

m, menu = int(sys.argv[1]), sys.argv[2]
Ls = [int(x) for x in sys.argv[3].split(",")]
total = float(sys.argv[4]) if len(sys.argv) > 4 else 2e8
q = gen.make_query(m)
rng = np.random.default_rng(7)
if menu != "plan":
    os.environ["SW_FORCE_MENU"] = menu
for L in Ls:
    n = int(total // L)
    res = rng.integers(0, 20, size=n * L, dtype=np.uint8)
    off = np.arange(n + 1, dtype=np.int64) * L
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(res, off)
        sw.search(1 << 30)
        sw.search(1 << 30)
        ms = sw.kernel_ms()["search_ms"]
    g = m * n * L / ms / 1e6
    print(f"m={m} menu={menu} len={L} n={n} kernel={ms:.2f} ms GCUPS={g:.0f} cells/clk/GPU={g / 1.965:.0f}", flush=True)
