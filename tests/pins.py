"""Independent references that PIN the oracle (test-only; SURVEY.md §8(c) "What pins each part").

None of these re-types Eq.(1): each is a different definition or a textbook routine that
Eq.(1) must reduce to.
  * brute_force_local  — enumerate every local alignment (all substring pairs, every
                         M/I/D column string, every open/extend choice of each gap column).
  * wsb_local          — cubic Waterman-Smith-Beyer general-gap DP with g(k) = rho + (k-1) sigma.
  * lcs_length         — longest common subsequence (textbook O(mn) DP).
  * longest_common_substring
  * max_ungapped_segment — Kadane's maximum-subarray over every diagonal.
"""
from __future__ import annotations

import itertools


def brute_force_local(q, d, W, rho, sigma, reopen=True):
    """max(0, best score over all local alignments of q and d).

    An alignment of q[a:b] with d[c:e] is a string of columns M (q_i with d_j), D (q_i
    against a gap: vertical move) and I (d_j against a gap: horizontal move).  Each gap
    column either opens a gap (cost rho) or — only directly after a gap column of the same
    direction — extends it (cost sigma).  With reopen=False a gap column after a
    same-direction gap column must extend (maximal-run affine cost rho + (k-1) sigma).
    Every path from every start is enumerated explicitly (depth-first); every prefix is
    itself an alignment ending at that cell.
    """
    m, n = len(q), len(d)
    best = 0

    def dfs(i, j, prev, score):
        nonlocal best
        if score > best:
            best = score
        if i < m and j < n:
            dfs(i + 1, j + 1, "M", score + int(W[q[i]][d[j]]))
        for mv, di, dj in (("D", 1, 0), ("I", 0, 1)):
            if i + di <= m and j + dj <= n:
                if prev == mv:
                    dfs(i + di, j + dj, mv, score - sigma)
                    if reopen:
                        dfs(i + di, j + dj, mv, score - rho)
                else:
                    dfs(i + di, j + dj, mv, score - rho)

    for a in range(m):
        for c in range(n):
            # an alignment must contain at least one column; start with any column type
            dfs(a, c, None, 0)
    return best


def wsb_local(q, d, W, rho, sigma):
    """Waterman-Smith-Beyer local alignment with general gap function g(k) = rho + (k-1) sigma.

    H[i][j] = max(0, H[i-1][j-1] + w, max_k H[i][j-k] - g(k), max_k H[i-k][j] - g(k)); O(mn(m+n)).
    """
    m, n = len(q), len(d)
    g = lambda k: rho + (k - 1) * sigma
    H = [[0] * (n + 1) for _ in range(m + 1)]
    best = 0
    for i in range(1, m + 1):
        for j in range(1, n + 1):
            v = H[i - 1][j - 1] + int(W[q[i - 1]][d[j - 1]])
            for k in range(1, j + 1):
                v = max(v, H[i][j - k] - g(k))
            for k in range(1, i + 1):
                v = max(v, H[i - k][j] - g(k))
            H[i][j] = max(0, v)
            best = max(best, H[i][j])
    return best


def lcs_length(a, b):
    m, n = len(a), len(b)
    L = [[0] * (n + 1) for _ in range(m + 1)]
    for i in range(1, m + 1):
        for j in range(1, n + 1):
            L[i][j] = L[i - 1][j - 1] + 1 if a[i - 1] == b[j - 1] else max(L[i - 1][j], L[i][j - 1])
    return L[m][n]


def longest_common_substring(a, b):
    best = 0
    for i in range(len(a)):
        for j in range(len(b)):
            k = 0
            while i + k < len(a) and j + k < len(b) and a[i + k] == b[j + k]:
                k += 1
            best = max(best, k)
    return best


def max_ungapped_segment(q, d, W):
    """max(0, max over diagonals of the maximum-sum contiguous run) — Kadane per diagonal."""
    m, n = len(q), len(d)
    best = 0
    for off in range(-(m - 1), n):
        cur = 0
        for i in range(m):
            j = i + off
            if 0 <= j < n:
                cur = max(0, cur + int(W[q[i]][d[j]]))
                best = max(best, cur)
    return best


def identity_matrix(A, match=1, mismatch=0):
    return [[match if a == b else mismatch for b in range(A)] for a in range(A)]


def all_strings(alpha, max_len):
    for L in range(max_len + 1):
        for t in itertools.product(alpha, repeat=L):
            yield list(t)
