"""CPU oracle for the Smith-Waterman database-search hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with the CUDA path
(``paper_conf_ipps_hainscobr11_b200``) and never imports it.

Contents
  * ``scores(...)``        — ctypes front-end of ``sw_oracle.c`` (scalar Eq.(1), int32,
                             OpenMP over database sequences).
  * ``eq1_tables(...)``    — Eq.(1) written out as full m x n E/F/H tables in plain Python
                             (tiny inputs), the definition in the paper's order/notation.

Eq.(1), §II (reading c1 of DESIGN.md):
    E[i][j] = max(E[i][j-1] - sigma, H[i][j-1] - rho)
    F[i][j] = max(F[i-1][j] - sigma, H[i-1][j] - rho)
    H[i][j] = max(0, E[i][j], F[i][j], H[i-1][j-1] + w(q_i, d_j))
    score = max_{i,j} H[i][j]            ("maximum score in table H", L12)
Boundary (reading c4): H[0][*] = H[*][0] = 0, E[*][0] = F[0][*] = -inf.

Every function here is pinned by tests/test_oracle_pins.py (brute force, cubic WSB DP,
Durbin Fig.2.5, LCS / longest-common-substring / Kadane special cases, invariants).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sw_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

NEG_INF = -(1 << 60)


def build(force: bool = False) -> str:
    """Compile sw_oracle.c with gcc -O2 -fopenmp (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.sw_oracle_scores.restype = ctypes.c_int
        L.sw_oracle_scores.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int32,
                                       ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                                       ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p]
        L.sw_oracle_pair.restype = ctypes.c_int32
        L.sw_oracle_pair.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64,
                                     ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32]
        L.sw_oracle_max_threads.restype = ctypes.c_int
        _lib = L
    return _lib


def max_threads() -> int:
    return int(lib().sw_oracle_max_threads())


def scores(query, matrix, rho: int, sigma: int, residues, offsets, threads: int = 0) -> np.ndarray:
    """Eq.(1) score of `query` against every CSR database sequence (int32, caller order)."""
    q = np.ascontiguousarray(query, dtype=np.uint8)
    W = np.ascontiguousarray(matrix, dtype=np.int8)
    A = W.shape[0]
    assert W.shape == (A, A)
    res = np.ascontiguousarray(residues, dtype=np.uint8)
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    N = off.shape[0] - 1
    out = np.zeros(max(N, 0), dtype=np.int32)
    if res.size == 0:
        res = np.zeros(1, dtype=np.uint8)
    rc = lib().sw_oracle_scores(q.ctypes.data, int(q.shape[0]), W.ctypes.data, int(A), int(rho), int(sigma),
                                res.ctypes.data, off.ctypes.data, int(N), int(threads), out.ctypes.data)
    if rc != 0:
        raise RuntimeError("sw_oracle_scores failed")
    return out


def pair(q, d, matrix, rho: int, sigma: int) -> int:
    q = np.ascontiguousarray(q, dtype=np.uint8)
    d = np.ascontiguousarray(d, dtype=np.uint8)
    W = np.ascontiguousarray(matrix, dtype=np.int8)
    qq = q if q.size else np.zeros(1, np.uint8)
    dd = d if d.size else np.zeros(1, np.uint8)
    return int(lib().sw_oracle_pair(qq.ctypes.data, int(q.shape[0]), dd.ctypes.data, int(d.shape[0]),
                                    W.ctypes.data, int(W.shape[0]), int(rho), int(sigma)))


def eq1_tables(q, d, matrix, rho: int, sigma: int, e0: int = NEG_INF, f0: int = NEG_INF):
    """Eq.(1) as full (m+1) x (n+1) tables E, F, H (plain Python ints; tiny inputs).

    e0 / f0 are the E[*][0] / F[0][*] boundary values (reading c4 says any value <= 0
    gives the same H; the default is -inf)."""
    m, n = len(q), len(d)
    E = [[e0] * (n + 1) for _ in range(m + 1)]
    F = [[f0] * (n + 1) for _ in range(m + 1)]
    H = [[0] * (n + 1) for _ in range(m + 1)]
    for i in range(1, m + 1):
        for j in range(1, n + 1):
            E[i][j] = max(E[i][j - 1] - sigma, H[i][j - 1] - rho)
            F[i][j] = max(F[i - 1][j] - sigma, H[i - 1][j] - rho)
            H[i][j] = max(0, E[i][j], F[i][j], H[i - 1][j - 1] + int(matrix[q[i - 1]][d[j - 1]]))
    return E, F, H


def eq1_score(q, d, matrix, rho: int, sigma: int, **kw) -> int:
    _, _, H = eq1_tables(q, d, matrix, rho, sigma, **kw)
    return max(max(row) for row in H)
