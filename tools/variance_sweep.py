"""Length-variance workload (Fig.2, §II-C): random
databases of N sequences with log-normal lengths, standard deviation swept (the mean grows
with it, "the mean to varies from 1000 to ..."), query of length 567; GCUPS of the short-
sequence (inter-task, T = inf) path and of the long-sequence (intra-task, T = 0) path.
The paper's claim: the inter-task kernel is very sensitive to the variance, the intra-task
kernel is not.   usage: python tools/variance_sweep.py [N=16384]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
q = gen.make_query(567)
for k, std in enumerate([100, 250, 500, 1000, 2000, 4000]):
    mean = 1000.0 + std
    s2 = np.log1p((std / mean) ** 2)
    mu = np.log(mean) - s2 / 2
    idx = np.arange(N, dtype=np.uint64)
    z = gen.normal(50 + k, "len", idx)
    lens = np.clip(np.rint(np.exp(mu + np.sqrt(s2) * z)), 2, 60000).astype(np.int64)
    db = gen.build_database(lens, 50 + k, None)
    cells = 567 * int(lens.sum())
    out = {"std": std, "mean": round(float(lens.mean()), 1), "max": int(lens.max()), "n": N}
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        for name, T in (("short_path", 1 << 30), ("long_path", 0), ("auto", -1)):
            sw.search(T)
            sw.search(T)
            ms = sw.kernel_ms()["search_ms"]
            out[name + "_gcups"] = round(cells / ms / 1e6, 1)
        out["auto_T"] = sw.last_threshold()
    print(json.dumps(out), flush=True)
