"""Long-path tail probe: kernel time of the long subset (n >= T) of C2, with and without its k
longest sequences, for T-mode overrides given as env settings.
usage: python tools/long_tail_probe.py m T "ENV=V;ENV=V,..." """
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

m, T = int(sys.argv[1]), int(sys.argv[2])
variants = sys.argv[3].split(",") if len(sys.argv) > 3 else [""]
lens = gen.sp_lengths(540_000, seed=2)
db = gen.build_database(lens, 2, None)
L = db.lengths
q = gen.make_query(m)
order = np.argsort(-L, kind="stable")
for drop in (0, 2, 8, 32):
    idx = np.sort(order[drop:][L[order[drop:]] >= T])
    off = np.concatenate([[0], np.cumsum(L[idx])]).astype(np.int64)
    res = np.concatenate([db.residues[db.offsets[i]:db.offsets[i + 1]] for i in idx])
    for v in variants:
        env = dict(kv.split("=") for kv in v.split(";") if kv)
        old = {k: os.environ.get(k) for k in env}
        os.environ.update(env)
        with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
            sw.load_db(res, off)
            sw.search(T)
            sw.search(T)
            ms = sw.kernel_ms()["search_ms"]
        for k, val in old.items():
            if val is None:
                os.environ.pop(k)
            else:
                os.environ[k] = val
        print(f"m={m} T={T} drop_longest={drop} seqs={idx.size} max={L[idx].max()} env={v or '-'} "
              f"ms={ms:.3f} GCUPS={m * int(L[idx].sum()) / ms / 1e6:.0f}", flush=True)
