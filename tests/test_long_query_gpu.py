"""Long queries (query length up to the ABI limit, not only what one CTA's
shared memory can hold as a query profile).  When the smallest query-profile image does not
fit (protein queries above ~8.9k residues), every pair runs in T-mode — the transposed kernel
that streams the query and builds substitution tables per database strip — and the flagged
sequences are recomputed by T-mode's 32-bit instantiation.
SW_LONG_QUERY=1 forces the mode for short queries so that every part of it (short and long
database sequences, empty ones, the 32-bit recompute, WIDE penalties) is covered cheaply.
Bit-exact against the oracle (§II Eq.(1))."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM45, BLOSUM62

pytestmark = pytest.mark.gpu


def _search(q, W, rho, sigma, db, T, env=None, batch=None):
    old = {k: os.environ.get(k) for k in (env or {})}
    os.environ.update({k: str(v) for k, v in (env or {}).items()})
    try:
        with swp.SmithWaterman(q, W, rho, sigma) as sw:
            sw.load_db(db.residues, db.offsets)
            out = sw.search(T) if batch is None else sw.search_batch(batch, T)
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


@pytest.mark.parametrize("m", [9000, 20000])
def test_long_protein_query(m):
    rng = np.random.default_rng(m)
    q = gen.make_query(m, seed=m)
    lens = np.concatenate([[0, 1, 47, 48, 49, 511, 512, 513, 3072, 12000], rng.integers(0, 800, size=120)])
    db = gen.build_database(lens.astype(np.int64), 31, [q], alphabet_extra=True)
    ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
    for T in (0, 3072, 1 << 30):
        got, st = _search(q, BLOSUM62, 10, 2, db, T)
        _check(got, ref, f"m={m} T={T}")
        assert st["long_seqs"] == db.num_seqs   # long-query mode: every pair in T-mode


@pytest.mark.parametrize("m", [1, 37, 700, 3000])
def test_forced_long_query_mode(m):
    rng = np.random.default_rng(100 + m)
    q = gen.make_query(m, seed=5 + m)
    lens = np.concatenate([np.arange(0, 40), rng.integers(40, 1200, size=100), [5000, 20000]])
    db = gen.build_database(lens.astype(np.int64), 33, [q], alphabet_extra=True)
    ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
    got, st = _search(q, BLOSUM62, 10, 2, db, 3072, {"SW_LONG_QUERY": 1})
    _check(got, ref, f"forced long-query m={m}")
    assert st["long_seqs"] == db.num_seqs
    # batch with the auto threshold (ignored in this mode)
    qs = [q, gen.make_query(max(1, m // 2), seed=9)]
    got, _ = _search(q, BLOSUM62, 10, 2, db, swp.SW_AUTO_THRESHOLD, {"SW_LONG_QUERY": 1}, batch=qs)
    for k, qq in enumerate(qs):
        _check(got[k], oracle.scores(qq, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0), f"batch q{k}")


@pytest.mark.parametrize("rho,env", [(10, {}), (200, {}), (20000, {}), (10, {"SW_T_GANG": "3"})])
def test_long_query_recompute_s32(rho, env):
    """Self-copies of a 9000-residue query under BLOSUM45 overflow the 16-bit lanes: the
    flagged sequences go through T-mode's 32-bit instantiation (WIDE for rho = 200, clamped
    16-bit penalties for rho = 20000)."""
    q = gen.make_query(9000, seed=3)
    rng = np.random.default_rng(rho)
    seqs = [rng.integers(0, 20, size=int(n)).astype(np.uint8) for n in rng.integers(0, 1500, size=40)]
    seqs += [q.copy(), q[:4000].copy(), np.concatenate([q[:5000], q[2000:7000]]), q[::-1].copy()]
    off = np.concatenate([[0], np.cumsum([s.size for s in seqs])]).astype(np.int64)
    db = gen.Database(np.concatenate(seqs), off, np.arange(len(seqs)))
    ref = oracle.scores(q, BLOSUM45, rho, 1, db.residues, db.offsets, threads=0)
    assert ref.max() > 32767
    got, st = _search(q, BLOSUM45, rho, 1, db, 3072, env)
    _check(got, ref, f"long-query recompute rho={rho} env={env}")
    assert st["recomputed_s32"] >= 2
