"""Pins of the CPU oracle against things other than itself (SURVEY.md §8(c) "What pins each part").

Each pin targets a plausible mistake: a dropped E or F term (brute force / WSB with gaps),
a wrong sign or index (Durbin's worked example, LCS, longest common substring), a missing
0-clamp (all-negative matrices), a transposed operand (asymmetric matrices against brute
force), a wrong boundary (c4 init invariance)."""
import os
import random

import numpy as np
import pytest

import oracle
from pins import (brute_force_local, identity_matrix, lcs_length, longest_common_substring,
                  max_ungapped_segment, wsb_local)
from workloads.matrices import ALPHABET, BLOSUM45, BLOSUM50, BLOSUM62, encode

HERE = os.path.dirname(os.path.abspath(__file__))


def _golden(name):
    vals = {}
    with open(os.path.join(HERE, "golden", name)) as f:
        for line in f:
            t = line.split()
            if t and not t[0].startswith("#") and t[0] not in ("row", "diag"):
                vals[t[0]] = t[1]
    return vals


def _rand_matrix(rng, A, lo=-4, hi=6, symmetric=False):
    M = [[rng.randint(lo, hi) for _ in range(A)] for _ in range(A)]
    if symmetric:
        for a in range(A):
            for b in range(a):
                M[a][b] = M[b][a]
    return M


def _all_three(q, d, W, rho, sigma):
    W8 = np.array(W, dtype=np.int8)
    return (oracle.pair(q, d, W8, rho, sigma), oracle.eq1_score(q, d, W, rho, sigma))


# --------------------------------------------------------------------------- worked example
def test_durbin_fig2_5():
    g = _golden("durbin_fig2_5.txt")
    q, d = encode(g["query"]), encode(g["subject"])
    W = {"BLOSUM50": BLOSUM50}[g["matrix"]]
    rho, sigma, want = int(g["gap_open"]), int(g["gap_extend"]), int(g["score"])
    assert oracle.pair(q, d, W, rho, sigma) == want
    assert oracle.eq1_score(list(q), list(d), W, rho, sigma) == want
    # the batch entry point agrees
    res = np.concatenate([d, q])
    off = np.array([0, len(d), len(d) + len(q)], dtype=np.int64)
    s = oracle.scores(q, W, rho, sigma, res, off, threads=2)
    assert s[0] == want


def test_durbin_pair_other_penalties_vs_brute_force():
    q, d = list(encode("HEAGAWGHEE")), list(encode("PAWHEAE"))
    for rho, sigma in [(10, 2), (12, 2), (10, 1), (5, 1), (0, 0), (8, 8)]:
        want = wsb_local(q, d, BLOSUM50, rho, sigma)
        assert oracle.pair(q, d, BLOSUM50, rho, sigma) == want
        # symmetric matrix: swapping q and d does not change the score
        assert oracle.pair(d, q, BLOSUM50, rho, sigma) == want


# --------------------------------------------------------------------------- brute force
def test_brute_force_tiny_random():
    rng = random.Random(1234)
    for case in range(400):
        A = rng.randint(2, 4)
        W = _rand_matrix(rng, A, -5, 6, symmetric=(case % 2 == 0))
        m, n = rng.randint(0, 4), rng.randint(0, 4)
        q = [rng.randrange(A) for _ in range(m)]
        d = [rng.randrange(A) for _ in range(n)]
        rho, sigma = rng.randint(0, 12), rng.randint(0, 14)
        want = brute_force_local(q, d, W, rho, sigma)
        c, py = _all_three(q, d, W, rho, sigma)
        assert c == want and py == want, (q, d, W, rho, sigma, want, c, py)


def test_brute_force_maximal_runs_when_extend_is_cheaper():
    """For sigma <= rho reopening never helps: the classic maximal-run affine definition."""
    rng = random.Random(99)
    for _ in range(200):
        A = 3
        W = _rand_matrix(rng, A, -4, 5)
        q = [rng.randrange(A) for _ in range(rng.randint(1, 4))]
        d = [rng.randrange(A) for _ in range(rng.randint(1, 4))]
        sigma = rng.randint(0, 6)
        rho = sigma + rng.randint(0, 8)
        want = brute_force_local(q, d, W, rho, sigma, reopen=False)
        assert oracle.pair(q, d, np.array(W, np.int8), rho, sigma) == want


# --------------------------------------------------------------------------- cubic WSB DP
def test_wsb_random_medium():
    rng = random.Random(7)
    for case in range(60):
        A = 24
        W = BLOSUM62 if case % 3 else _rand_matrix(rng, A, -6, 8)
        q = [rng.randrange(20) for _ in range(rng.randint(1, 40))]
        d = [rng.randrange(20) for _ in range(rng.randint(0, 40))]
        rho, sigma = rng.choice([(10, 2), (12, 2), (3, 7), (0, 0), (1, 1), (20, 1)])
        assert oracle.pair(q, d, np.array(W, np.int8), rho, sigma) == wsb_local(q, d, W, rho, sigma)


def test_wsb_planted_homologue():
    rng = random.Random(11)
    q = [rng.randrange(20) for _ in range(120)]
    d = [rng.randrange(20) for _ in range(30)] + q[20:90] + [rng.randrange(20) for _ in range(25)]
    del d[60:63]          # a deletion
    d[70:70] = [3, 4]     # an insertion
    for W, rho, sigma in [(BLOSUM62, 10, 2), (BLOSUM45, 10, 2), (BLOSUM62, 12, 2)]:
        want = wsb_local(q, d, W, rho, sigma)
        assert want > 100
        assert oracle.pair(q, d, W, rho, sigma) == want


# --------------------------------------------------------------------------- textbook special cases
def test_lcs_special_case():
    """rho = sigma = 0 and w = [a == b]: the score is the LCS length."""
    rng = random.Random(5)
    W = np.array(identity_matrix(4, 1, 0), np.int8)
    for _ in range(200):
        a = [rng.randrange(4) for _ in range(rng.randint(0, 30))]
        b = [rng.randrange(4) for _ in range(rng.randint(0, 30))]
        assert oracle.pair(a, b, W, 0, 0) == lcs_length(a, b)


def test_longest_common_substring_special_case():
    rng = random.Random(6)
    W = np.array(identity_matrix(4, 1, -100), np.int8)
    for _ in range(200):
        a = [rng.randrange(4) for _ in range(rng.randint(0, 30))]
        b = [rng.randrange(4) for _ in range(rng.randint(0, 30))]
        assert oracle.pair(a, b, W, 100, 100) == longest_common_substring(a, b)


def test_ungapped_kadane_special_case():
    rng = random.Random(8)
    for _ in range(150):
        a = [rng.randrange(20) for _ in range(rng.randint(1, 40))]
        b = [rng.randrange(20) for _ in range(rng.randint(1, 40))]
        big = 11 * max(len(a), len(b)) + 1
        assert oracle.pair(a, b, BLOSUM62, big, big) == max_ungapped_segment(a, b, BLOSUM62)


def test_single_residue_query():
    rng = random.Random(9)
    for _ in range(100):
        a = rng.randrange(24)
        d = [rng.randrange(24) for _ in range(rng.randint(0, 50))]
        want = max([0] + [int(BLOSUM62[a][x]) for x in d])
        assert oracle.pair([a], d, BLOSUM62, 10, 2) == want


def test_all_negative_matrix_scores_zero():
    W = np.full((4, 4), -3, np.int8)
    assert oracle.pair([0, 1, 2, 3], [0, 1, 2, 3], W, 0, 0) == 0


def test_asymmetric_matrix_orientation():
    """w is indexed [query symbol][db symbol] (reading c5); a transposed lookup fails this."""
    W = np.array([[0, 9], [-9, 0]], np.int8)
    assert oracle.pair([0], [1], W, 5, 5) == 9
    assert oracle.pair([1], [0], W, 5, 5) == 0
    assert brute_force_local([0], [1], W, 5, 5) == 9


# --------------------------------------------------------------------------- invariants
def _self_score_condition(W, letters):
    for a in letters:
        if W[a][a] <= 0:
            return False
        for b in letters:
            if 2 * int(W[a][b]) > int(W[a][a]) + int(W[b][b]):
                return False
    return True


def test_self_score_is_diagonal_sum():
    letters = list(range(20))
    assert _self_score_condition(BLOSUM62, letters)
    rng = random.Random(10)
    for _ in range(50):
        s = [rng.choice(letters) for _ in range(rng.randint(1, 200))]
        want = sum(int(BLOSUM62[x][x]) for x in s)
        assert oracle.pair(s, s, BLOSUM62, 10, 2) == want


def test_invariants_random():
    rng = random.Random(12)
    for _ in range(150):
        q = [rng.randrange(20) for _ in range(rng.randint(1, 35))]
        d = [rng.randrange(20) for _ in range(rng.randint(1, 35))]
        rho, sigma = rng.randint(0, 12), rng.randint(0, 4)
        s = oracle.pair(q, d, BLOSUM62, rho, sigma)
        assert 0 <= s <= min(len(q), len(d)) * 11
        assert oracle.pair(d, q, BLOSUM62, rho, sigma) == s                        # symmetry
        assert oracle.pair(q, d, BLOSUM62, rho + 1, sigma) <= s                   # monotone in rho
        assert oracle.pair(q, d, BLOSUM62, rho, sigma + 1) <= s                   # monotone in sigma
        x = [rng.randrange(20) for _ in range(rng.randint(0, 10))]
        y = [rng.randrange(20) for _ in range(rng.randint(0, 10))]
        assert oracle.pair(q, x + d + y, BLOSUM62, rho, sigma) >= s               # superstring
        d2 = [rng.randrange(20) for _ in range(rng.randint(1, 20))]
        assert oracle.pair(q, d + d2, BLOSUM62, rho, sigma) >= max(s, oracle.pair(q, d2, BLOSUM62, rho, sigma))


def test_boundary_init_invariance_c4():
    rng = random.Random(13)
    for _ in range(200):
        A = 4
        W = _rand_matrix(rng, A, -4, 5)
        q = [rng.randrange(A) for _ in range(rng.randint(1, 8))]
        d = [rng.randrange(A) for _ in range(rng.randint(1, 8))]
        rho, sigma = rng.randint(0, 10), rng.randint(0, 10)
        _, _, H0 = oracle.eq1_tables(q, d, W, rho, sigma)
        for e0, f0 in [(0, 0), (-rho, -rho), (0, -rho), (-1000, 0)]:
            _, _, H1 = oracle.eq1_tables(q, d, W, rho, sigma, e0=e0, f0=f0)
            assert H1 == H0


def test_homopolymer_beyond_int16():
    """W^k vs W^k' scores exactly min(k, k') * 11 under BLOSUM62 (overflow pins, §8(c) 6)."""
    w = ALPHABET.index("W")
    for k, k2 in [(2900, 3100), (3000, 3100), (3100, 3000)]:
        assert oracle.pair([w] * k, [w] * k2, BLOSUM62, 10, 2) == min(k, k2) * 11


def test_batch_matches_pairs_and_threads():
    rng = np.random.default_rng(3)
    lens = rng.integers(0, 300, size=200)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    res = rng.integers(0, 24, size=int(off[-1])).astype(np.uint8)
    q = rng.integers(0, 24, size=77).astype(np.uint8)
    s1 = oracle.scores(q, BLOSUM62, 10, 2, res, off, threads=1)
    s4 = oracle.scores(q, BLOSUM62, 10, 2, res, off, threads=4)
    assert np.array_equal(s1, s4)
    for k in range(0, 200, 17):
        assert s1[k] == oracle.pair(q, res[off[k]:off[k + 1]], BLOSUM62, 10, 2)
    assert s1[lens == 0].sum() == 0
