"""Drive searches of the LONG subset (n >= T) of a config's database with one query, the
isolated long-regime launch of the threshold sweeps (for ncu captures of k_search_t).
usage: python tools/profile_long.py [query_len=567] [T=3072] [reps=3] [config=C2] [env=K=V;...] [top:K|drop:K]
(top:K keeps only the K longest sequences of the subset, drop:K removes them)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

m = int(sys.argv[1]) if len(sys.argv) > 1 else 567
T = int(sys.argv[2]) if len(sys.argv) > 2 else 3072
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
cfg = sys.argv[4] if len(sys.argv) > 4 else "C2"
if len(sys.argv) > 5 and sys.argv[5]:
    os.environ.update(dict(kv.split("=") for kv in sys.argv[5].split(";") if kv))
if cfg == "C3":
    lens = gen.long_lengths(4096, seed=3)
    db = gen.build_database(lens, 3, None)
else:
    lens = gen.sp_lengths(540_000, seed=2)
    db = gen.build_database(lens, 2, None)
L = db.lengths
idx = np.nonzero(L >= T)[0]
if len(sys.argv) > 6 and sys.argv[6]:
    mode, k = sys.argv[6].split(":")
    order = idx[np.argsort(-L[idx], kind="stable")]
    idx = np.sort(order[:int(k)] if mode == "top" else order[int(k):])
off = np.concatenate([[0], np.cumsum(L[idx])]).astype(np.int64)
res = np.concatenate([db.residues[db.offsets[i]:db.offsets[i + 1]] for i in idx])
if os.environ.get("SW_PROBE_EXTRA"):   # extra synthetic sequences (e.g. an outlier pair for the row scan)
    ext = [int(x) for x in os.environ["SW_PROBE_EXTRA"].split(",")]
    rng = np.random.default_rng(11)
    res = np.concatenate([res] + [rng.integers(0, 20, size=n).astype(np.uint8) for n in ext])
    off = np.concatenate([off, off[-1] + np.cumsum(ext)]).astype(np.int64)
    idx = np.concatenate([idx, np.zeros(len(ext), np.int64)])
q = gen.make_query(m)
if os.environ.get("SW_LIB"):          # A/B against another build of the library
    swp.load_library(os.environ["SW_LIB"])
with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
    sw.load_db(res, off)
    for _ in range(reps):
        sw.search(T)
        ms = sw.kernel_ms()["search_ms"]
        print(f"{cfg} long subset n>={T}: {idx.size} seqs, {int(off[-1])} residues, m={m}: {ms:.3f} ms "
              f"{m * int(off[-1]) / ms / 1e6:.0f} GCUPS", flush=True)
