"""Parity on the f2 workload shapes: the length-variance databases of
PAPER.md Fig.2 (L16 §II-C; lengths to 60,000, standard deviation to 4000) and the Table II
databases (L28-L30; 0.06-0.56 % of the sequences over 3072), subsampled to 2,000 sequences,
through both regimes, the automatic threshold and both long-sequence paths, bit-exact against
the oracle (Eq.(1), L12 §II)."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM62

pytestmark = pytest.mark.gpu


def _run(q, db, T, mode=None):
    if mode:
        os.environ["SW_LONG_MODE"] = mode
    try:
        with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
            sw.load_db(db.residues, db.offsets)
            return sw.search(T)
    finally:
        os.environ.pop("SW_LONG_MODE", None)


def _check(got, ref, what):
    bad = np.nonzero(got != ref)[0]
    assert bad.size == 0, f"{what}: {bad.size} mismatches, first {bad[:6]}"


@pytest.mark.parametrize("std", [250, 4000])
def test_variance_db_parity(std):
    k = gen.VARIANCE_STDS.index(std)
    lens = gen.variance_lengths(16384, std, seed=50 + k)
    sel = np.arange(0, 16384, 8)[:2000]
    db = gen.build_database(lens, 50 + k, None, sel=sel)
    assert db.num_seqs == 2000
    for m in (144, 567, 3564):
        q = gen.make_query(m)
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
        for T, mode in ((0, None), (3072, None), (3072, "team"), (1 << 30, None), (-1, None)):
            _check(_run(q, db, T, mode), ref, f"std={std} m={m} T={T} mode={mode}")


@pytest.mark.parametrize("which", ["RefSeq Human", "TAIR"])
def test_table2_db_parity(which):
    k = [n for n, _ in gen.TABLE2].index(which)
    frac = gen.TABLE2[k][1]
    lens = gen.table2_lengths(200_000, frac, seed=70 + k)
    order = np.argsort(-lens, kind="stable")
    sel = np.unique(np.concatenate([order[:40], np.arange(0, 200_000, 100)]))   # the long tail + every 100th
    db = gen.build_database(lens, 70 + k, None, sel=sel)
    for m in (144, 1500):
        q = gen.make_query(m)
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
        for T, mode in ((3072, None), (3072, "team"), (1536, None), (-1, None)):
            _check(_run(q, db, T, mode), ref, f"{which} m={m} T={T} mode={mode}")
