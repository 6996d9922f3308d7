"""Table II analog (Table II, reading c19): synthetic
databases whose fraction of sequences over T = 3072 matches the six real databases of Table II
(Ensembl Dog 0.53 %, Ensembl Rat 0.35 %, RefSeq Human 0.56 %, RefSeq Mouse 0.54 %, TAIR 0.06 %,
Swiss-Prot 0.12 %).  Lengths are log-normal with Swiss-Prot's median (mu = 5.5219) and a
sigma solved so that P(n >= 3072) hits the target.  For each database, the C2 query set is
searched with the long sequences on the T-mode kernel (default), on the query-strip team kernel
(the paper's intra-task orientation, SW_LONG_MODE=team), and with the automatic threshold.
GCUPS = cells / device time (CUDA events around one batched search, queries on 4 streams).
usage: python tools/table2_sweep.py [N=200000]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
from scipy.stats import norm  # noqa: E402

import paper_conf_ipps_hainscobr11_b200 as swp  # noqa: E402
from workloads import gen  # noqa: E402
from workloads.matrices import BLOSUM62  # noqa: E402

N = int(sys.argv[1]) if len(sys.argv) > 1 else 200000
MU = 5.5219
TABLE2 = [("Ensembl Dog", 0.0053), ("Ensembl Rat", 0.0035), ("RefSeq Human", 0.0056),
          ("RefSeq Mouse", 0.0054), ("TAIR", 0.0006), ("Swiss-Prot", 0.0012)]
QS = [gen.make_query(m) for m in (144, 375, 729, 1500, 5478)]


def timed(sw, out, T, reps=2):
    st = torch.cuda.current_stream()
    sw.search_batch_into(QS, out.data_ptr(), T, st.cuda_stream)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(reps):
        sw.search_batch_into(QS, out.data_ptr(), T, st.cuda_stream)
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


for k, (name, frac) in enumerate(TABLE2):
    sigma = (np.log(3072.0) - MU) / norm.ppf(1.0 - frac)
    lens = gen.sp_lengths(N, seed=70 + k, mu=MU, sigma=float(sigma), tail_frac=0.0)
    db = gen.build_database(lens, 70 + k, None)
    cells = sum(int(q.size) for q in QS) * int(lens.sum())
    row = {"db": name, "target_pct_over_T": round(100 * frac, 2),
           "pct_over_T": round(100 * float((lens >= 3072).mean()), 3), "sigma": round(float(sigma), 4),
           "n": N, "residues": int(lens.sum()), "max_len": int(lens.max())}
    out = torch.zeros((len(QS), N), dtype=torch.int32, device="cuda")
    with swp.SmithWaterman(QS[0], BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        ref = None
        for label, T, env in (("tmode_T3072", 3072, None), ("team_T3072", 3072, "team"), ("auto", -1, None)):
            if env:
                os.environ["SW_LONG_MODE"] = env
            ms = timed(sw, out, T)
            os.environ.pop("SW_LONG_MODE", None)
            row[label + "_gcups"] = round(cells / ms / 1e6, 1)
            cur = out.cpu().numpy()
            if ref is None:
                ref = cur
            assert np.array_equal(ref, cur), label          # scores do not depend on T or the mode
        row["auto_T"] = sw.last_threshold()
    print(json.dumps(row), flush=True)
