"""GPU parity of the row-scan path (csrc/sw_scan.cu): the
longest long pairs computed one query row per cluster time step (max-plus prefix scan of the
horizontal gap term along the row, DSMEM hand-off between the cluster's CTAs), bit-exact
against the CPU oracle of Eq.(1) (§II).

SW_SCAN=N forces the scan for every long pair of >= N columns (up to kMaxScanItems = 4 pairs,
clusters of 1..16 CTAs of 4096 columns); the remaining long pairs take k_search_t's team
stream, whose queue then starts after the scanned pairs."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM45, BLOSUM62

pytestmark = pytest.mark.gpu


def _search(q, W, rho, sigma, db, T, env):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update({k: str(v) for k, v in env.items()})
    try:
        with swp.SmithWaterman(q, W, rho, sigma) as sw:
            sw.load_db(db.residues, db.offsets)
            out = sw.search(T)
            st = sw.stats()
        return out, st
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _check(out, ref, db, what):
    bad = np.nonzero(out != ref)[0]
    assert bad.size == 0, (f"{what}: {bad.size} mismatches, first {bad[:8]} "
                           f"lens {np.diff(db.offsets)[bad[:8]]} got {out[bad[:8]]} want {ref[bad[:8]]}")


@pytest.mark.parametrize("m", [144, 567, 1500, 2999])
def test_scan_pairs_match_oracle(m):
    """Clusters of 9, 5, 3 and 1 CTAs (pairs of 35,213 / 20,000 / 9,000 / 4,000 columns) beside
    the team stream's pairs; both members of a pair differ in length (ragged pad columns)."""
    rng = np.random.default_rng(70 + m)
    lens = np.concatenate([[35213, 34100, 20000, 17000, 9000, 8100, 4000, 3100],
                           rng.integers(3073, 6000, size=6), rng.integers(0, 400, size=40)])
    db = gen.build_database(lens.astype(np.int64), 80 + m, None)
    q = gen.make_query(m, seed=90 + m)
    ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets)
    for T in (3072, 0):
        out, _ = _search(q, BLOSUM62, 10, 2, db, T, {"SW_LONG_MODE": "t", "SW_SCAN": "1"})
        _check(out, ref, db, f"m={m} T={T}")


@pytest.mark.parametrize("rho,sigma,W", [(5, 9, BLOSUM62), (14, 2, BLOSUM45), (3, 3, BLOSUM62), (11, 0, BLOSUM62)])
def test_scan_penalties(rho, sigma, W):
    """sigma > rho (close and reopen: the scan's sigma' = min(sigma, rho)), sigma = rho, sigma = 0
    and BLOSUM45."""
    rng = np.random.default_rng(rho * 31 + sigma)
    lens = np.concatenate([[21000, 12000, 7000, 4100], rng.integers(0, 300, size=20)])
    db = gen.build_database(lens.astype(np.int64), 7 + rho, None)
    q = gen.make_query(400, seed=rho + sigma)
    ref = oracle.scores(q, W, rho, sigma, db.residues, db.offsets)
    out, _ = _search(q, W, rho, sigma, db, 3000, {"SW_LONG_MODE": "t", "SW_SCAN": "1"})
    _check(out, ref, db, f"rho={rho} sigma={sigma}")


def test_scan_overflow_recompute():
    """A pair whose s16 score saturates (a 2,990-residue W homopolymer query against a sequence
    holding it): flagged by the scan kernel, recomputed exactly in 32 bits."""
    A = 24
    w_idx = 17   # W in the NCBI order ARNDCQEGHILKMFPSTWYVBZX*
    q = np.full(2990, w_idx, np.uint8)
    rng = np.random.default_rng(3)
    seqs = [rng.integers(0, 20, size=n).astype(np.uint8) for n in (20000, 18000, 5000, 300)]
    seqs[1][5000:5000 + 2990] = w_idx
    res = np.concatenate(seqs)
    off = np.concatenate([[0], np.cumsum([len(s) for s in seqs])]).astype(np.int64)

    class _Db:
        pass
    db = _Db()
    db.residues, db.offsets = res, off
    ref = oracle.scores(q, BLOSUM62, 10, 2, res, off)
    assert ref.max() > 32767 - 11
    out, st = _search(q, BLOSUM62, 10, 2, db, 3000, {"SW_LONG_MODE": "t", "SW_SCAN": "1"})
    _check(out, ref, db, "overflow")
    assert st["recomputed_s32"] >= 1
    del A


def test_scan_repeated_and_batched():
    """Repeated searches and a batch on one handle (the scan stream, its events and the kernel's
    cluster configuration are reused; the message slots are re-initialised per launch)."""
    rng = np.random.default_rng(5)
    lens = np.concatenate([[30000, 26000, 16500, 9000], rng.integers(0, 500, size=30)])
    db = gen.build_database(lens.astype(np.int64), 17, None)
    os.environ.update({"SW_LONG_MODE": "t", "SW_SCAN": "1"})
    try:
        qs = [gen.make_query(m, seed=m) for m in (200, 700, 1100)]
        refs = [oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets) for q in qs]
        with swp.SmithWaterman(qs[0], BLOSUM62, 10, 2) as sw:
            sw.load_db(db.residues, db.offsets)
            for k in range(3):
                _check(sw.search(3000), refs[0], db, f"repeat {k}")
            outb = sw.search_batch(qs, 3000)
            for k in range(3):
                _check(outb[k], refs[k], db, f"batch {k}")
    finally:
        os.environ.pop("SW_LONG_MODE", None)
        os.environ.pop("SW_SCAN", None)


def test_scan_chosen_automatically_for_an_outlier_pair():
    """No SW_SCAN: the planner scans pair 0 on its own when it is an outlier (its time alone
    bounds the launch and it has >= 1.5x the next pair's columns) — a 64,000 / 60,000-residue
    pair beside 3-8k sequences — with gangs / teams for the rest, the T-mode kernel as a
    programmatic dependent launch behind the scan."""
    rng = np.random.default_rng(99)
    lens = np.concatenate([[64000, 60000], rng.integers(3073, 8000, size=60), rng.integers(0, 300, size=30)])
    db = gen.build_database(lens.astype(np.int64), 123, None)
    for m in (300, 567):
        q = gen.make_query(m, seed=m + 7)
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets)
        out, _ = _search(q, BLOSUM62, 10, 2, db, 3072, {"SW_LONG_MODE": "t"})
        _check(out, ref, db, f"auto scan m={m}")
