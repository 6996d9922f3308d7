"""Any gap penalties rho, sigma >= 0 (§II: Eq.(1) puts no bound on them; SURVEY.md
§8(b)).  rho + max(w) > 127 does not fit the int8 profile entry w + rho: the WIDE kernels hold
w + c in the profile and add delta = rho - c per cell; penalties above 16384 are clamped for the
16-bit lanes with a lowered overflow flag (exact for every sequence below the flag, the rest
recomputed in 32 bits) — DESIGN.md "Integer widths".  Every case: bit-exact against the oracle,
both regimes and both long-sequence paths."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from pins import max_ungapped_segment
from workloads import gen
from workloads.matrices import BLOSUM45, BLOSUM62

pytestmark = pytest.mark.gpu


def _search(q, W, rho, sigma, db, T, env=None):
    old = {k: os.environ.get(k) for k in (env or {})}
    os.environ.update({k: str(v) for k, v in (env or {}).items()})
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


def _check(got, ref, what):
    bad = np.nonzero(got != ref)[0]
    assert bad.size == 0, f"{what}: {bad.size} mismatches, first {[(int(i), int(got[i]), int(ref[i])) for i in bad[:6]]}"


@pytest.mark.parametrize("rho,sigma", [(117, 2), (200, 300), (300, 1), (5000, 5000), (20000, 1), (1, 20000),
                                       (1_000_000, 1_000_000)])
def test_large_penalties_parity(rho, sigma):
    rng = np.random.default_rng(rho + sigma)
    lens = np.concatenate([rng.integers(0, 500, size=150), [3100, 4500, 9000]])
    db = gen.build_database(lens.astype(np.int64), 12, None, alphabet_extra=True)
    for m in (37, 300, 1500):
        q = gen.make_query(m, seed=m + 3)
        ref = oracle.scores(q, BLOSUM62, rho, sigma, db.residues, db.offsets, threads=0)
        for T in (0, 3072, 1 << 30):
            for mode in ("t", "team"):
                if T == 1 << 30 and mode == "team":
                    continue
                got, _ = _search(q, BLOSUM62, rho, sigma, db, T, {"SW_LONG_MODE": mode})
                _check(got, ref, f"rho={rho} sigma={sigma} m={m} T={T} mode={mode}")


def test_kadane_special_case():
    """rho, sigma >= m * max(w): no gap can pay, Eq.(1) reduces to the maximum ungapped segment
    (Kadane along every diagonal, SURVEY.md §8(c) pin 3) — rho far beyond the int8 profile."""
    rng = np.random.default_rng(77)
    lens = np.concatenate([rng.integers(0, 300, size=30), [3300]])
    db = gen.build_database(lens.astype(np.int64), 17, None)
    q = gen.make_query(200, seed=17)
    big = 200 * 11
    want = np.array([max_ungapped_segment(q, db.residues[db.offsets[k]:db.offsets[k + 1]], BLOSUM62)
                     for k in range(db.num_seqs)], np.int32)
    ref = oracle.scores(q, BLOSUM62, big, big, db.residues, db.offsets, threads=0)
    assert np.array_equal(ref, want)
    for T in (0, 1 << 30):
        got, _ = _search(q, BLOSUM62, big, big, db, T)
        _check(got, want, f"Kadane T={T}")


@pytest.mark.parametrize("rho", [200, 20000])
def test_wide_overflow_recompute(rho):
    """Self-copies of a 5478-residue query under BLOSUM45 score > 32767 (and > the clamped
    flag 16384): the WIDE s16 pass flags them and the WIDE 32-bit recompute decides."""
    q = gen.make_query(5478)
    rng = np.random.default_rng(rho)
    seqs = [rng.integers(0, 20, size=int(n)).astype(np.uint8) for n in rng.integers(10, 2000, size=30)]
    seqs += [q.copy(), q[:2500].copy(), np.concatenate([q[:3000], q[:3000]])]
    off = np.concatenate([[0], np.cumsum([s.size for s in seqs])]).astype(np.int64)
    db = gen.Database(np.concatenate(seqs), off, np.arange(len(seqs)))
    ref = oracle.scores(q, BLOSUM45, rho, 1, db.residues, db.offsets, threads=0)
    assert ref.max() > 16384
    for T in (0, 3072, 1 << 30):
        got, st = _search(q, BLOSUM45, rho, 1, db, T)
        _check(got, ref, f"wide self-copy rho={rho} T={T}")
        assert st["recomputed_s32"] >= 1
