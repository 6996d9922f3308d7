"""Threshold sweep (Fig.3 / Fig.5 analog): for each T, kernel time
of the whole search and of each regime in isolation (only that subset of the database).

usage: python tools/sweep_threshold.py C2|C3 query_len T1,T2,...   -> one JSON line per T"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

cfg, m = sys.argv[1], int(sys.argv[2])
Ts = [int(x) if x != "auto" else -1 for x in sys.argv[3].split(",")]
if cfg == "C3":
    lens = gen.long_lengths(4096, seed=3)
    db = gen.build_database(lens, 3, None)
else:
    lens = gen.sp_lengths(540_000, seed=2)
    db = gen.build_database(lens, 2, None)
L = db.lengths
q = gen.make_query(m)


def subset(mask):
    idx = np.nonzero(mask)[0]
    off = np.concatenate([[0], np.cumsum(L[idx])]).astype(np.int64)
    res = np.concatenate([db.residues[db.offsets[i]:db.offsets[i + 1]] for i in idx]) if idx.size else np.zeros(0, np.uint8)
    return res, off, int(L[idx].sum())


LAST_T = [None]
LAST_REGIME = [None]


def timed(res, off, T):
    if off.shape[0] <= 1 or off[-1] == 0:
        return 0.0
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(res, off)
        sw.search(T)
        sw.search(T)
        LAST_T[0] = sw.last_threshold()
        LAST_REGIME[0] = sw.regime_ms()
        return sw.kernel_ms()["search_ms"]


full_ms = {}
for T in Ts:
    t_all = timed(db.residues, db.offsets, T)
    reg = LAST_REGIME[0]
    auto = T < 0
    if auto:
        T = LAST_T[0]
    res_l, off_l, n_l = subset(L >= T)
    res_s, off_s, n_s = subset(L < T)
    t_l = timed(res_l, off_l, T)
    t_s = timed(res_s, off_s, T)
    line = {"config": cfg, "m": m, "T": T, "auto": auto, "frac_seqs_long": round(float((L >= T).mean()), 5),
            "frac_res_long": round(n_l / max(1, int(L.sum())), 5), "ms_total": round(t_all, 3),
            "gcups_total": round(m * int(L.sum()) / t_all / 1e6, 1) if t_all else None,
            "gcups_long_only": round(m * n_l / t_l / 1e6, 1) if t_l else None,
            "gcups_short_only": round(m * n_s / t_s / 1e6, 1) if t_s else None,
            # Fig.5b analog: time of the long-path (T-mode) launch in the combined search, which
            # runs concurrently with the short-sequence launch (share of the search interval)
            "long_kernel_ms": round(reg["long_ms"], 3) if reg else None,
            "pct_time_long_kernel": round(100 * reg["long_ms"] / reg["search_ms"], 1)
            if reg and reg["search_ms"] > 0 and not reg["fused_long_queries"] else None}
    if line["gcups_long_only"] and line["gcups_short_only"]:
        line["long_over_short"] = round(line["gcups_long_only"] / line["gcups_short_only"], 3)
    print(json.dumps(line), flush=True)
