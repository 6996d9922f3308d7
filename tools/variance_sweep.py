"""Length-variance workload (Fig.2, §II-C): random
databases of N sequences with log-normal lengths (workloads/gen.py variance_lengths: standard
deviation swept, mean 1000 + std), query of length 567; GCUPS of the short-sequence
(inter-task, T = inf) path, of the long-sequence (intra-task, T = 0) path, of fixed thresholds
and of the automatic threshold.  The paper's claim: the inter-task kernel is very sensitive to
the variance, the intra-task kernel is not.   usage: python tools/variance_sweep.py [N=16384] [m=567]"""
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
m = int(sys.argv[2]) if len(sys.argv) > 2 else 567
q = gen.make_query(m)
for k, std in enumerate(gen.VARIANCE_STDS):
    lens = gen.variance_lengths(N, std, seed=50 + k)
    db = gen.build_database(lens, 50 + k, None)
    cells = m * int(lens.sum())
    out = {"std": std, "mean": round(float(lens.mean()), 1), "max": int(lens.max()), "n": N, "m": m}
    fixed = {}
    ref = None
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        for name, T in (("short_path", 1 << 30), ("long_path", 0), ("T8192", 8192), ("T4096", 4096),
                        ("T3072", 3072), ("T2048", 2048), ("T1024", 1024), ("auto", -1)):
            got = sw.search(T)
            sw.search(T)
            ms = sw.kernel_ms()["search_ms"]
            out[name + "_gcups"] = round(cells / ms / 1e6, 1)
            if name != "auto":
                fixed[name] = out[name + "_gcups"]
            if ref is None:
                ref = got
            assert np.array_equal(ref, got), name
        out["auto_T"] = sw.last_threshold()
    best = max(fixed, key=fixed.get)
    out["best_fixed"] = best
    out["auto_over_best_fixed"] = round(out["auto_gcups"] / fixed[best], 4)
    out["long_over_short"] = round(out["long_path_gcups"] / out["short_path_gcups"], 4)
    print(json.dumps(out), flush=True)
