"""Randomised GPU parity (seeded, deterministic): the whole search API against the CPU oracle of
Eq.(1) (§II) over random scoring schemes and shapes — alphabets of 2-32 letters,
random (asymmetric) integer matrices, any rho / sigma (WIDE kernels and clamped 16-bit
penalties included), sigma > rho, random thresholds (both regimes, T-mode, gangs, row scans),
ragged and empty sequences, batches of queries — so that combinations no hand-written case
names are checked too."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp

pytestmark = pytest.mark.gpu

N_CASES = 96


def _case(seed):
    rng = np.random.default_rng(10_000 + seed)
    A = int(rng.choice([2, 4, 20, 24, 32]))
    lo, hi = int(rng.integers(-20, -1)), int(rng.integers(1, 20))
    W = rng.integers(lo, hi + 1, size=(A, A)).astype(np.int8)
    if rng.random() < 0.5:
        W = np.triu(W) + np.triu(W, 1).T   # symmetric half the time
    rho = int(rng.choice([0, 1, 5, 10, 40, 120, 300, 20000]))
    sigma = int(rng.choice([0, 1, 2, 7, 60, 500]))
    n = int(rng.integers(1, 300))
    kind = rng.random()
    if kind < 0.4:
        lens = rng.integers(0, 700, size=n)
    elif kind < 0.8:
        lens = np.concatenate([rng.integers(0, 500, size=n), rng.integers(2000, 9000, size=int(rng.integers(1, 8)))])
    else:
        lens = np.concatenate([rng.integers(0, 300, size=n), [int(rng.integers(16384, 24000))]])
    rng.shuffle(lens)
    res = rng.integers(0, A, size=int(lens.sum())).astype(np.uint8)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    nq = int(rng.integers(1, 4))
    qs = [rng.integers(0, A, size=int(rng.choice([1, 17, 144, 567, 1200, 2999, 3100]))).astype(np.uint8)
          for _ in range(nq)]
    T = int(rng.choice([0, 1, 100, 1000, 3072, 1 << 30]))
    env = {}
    r = rng.random()
    if r < 0.15:
        env["SW_SCAN"] = "1"
        env["SW_LONG_MODE"] = "t"
    elif r < 0.3:
        env["SW_T_GANG"] = "3"
        env["SW_LONG_MODE"] = "t"
    return A, W, rho, sigma, res, off, qs, T, env


@pytest.mark.parametrize("seed", range(N_CASES))
def test_fuzz_parity(seed):
    A, W, rho, sigma, res, off, qs, T, env = _case(seed)
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        with swp.SmithWaterman(qs[0], W, rho, sigma) as sw:
            sw.load_db(res, off)
            out = sw.search_batch(qs, T)
        for k, q in enumerate(qs):
            ref = oracle.scores(q, W, rho, sigma, res, off)
            bad = np.nonzero(out[k] != ref)[0]
            assert bad.size == 0, (f"seed={seed} A={A} rho={rho} sigma={sigma} T={T} env={env} m={q.size} "
                                   f"query {k}: {bad.size} mismatches, first {bad[:6]} lens "
                                   f"{np.diff(off)[bad[:6]]} got {out[k][bad[:6]]} want {ref[bad[:6]]}")
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
