"""Transcription checks of the substitution-matrix INPUTS (reading c7)."""
import os

import numpy as np

from workloads.matrices import ALPHABET, BLOSUM45, BLOSUM50, BLOSUM62, encode, decode

HERE = os.path.dirname(os.path.abspath(__file__))


def test_symmetric():
    for M in (BLOSUM45, BLOSUM50, BLOSUM62):
        assert M.shape == (24, 24)
        assert np.array_equal(M, M.T)


def test_blosum62_diagonal_and_extrema():
    diag = dict(A=4, R=5, N=6, D=6, C=9, Q=5, E=5, G=6, H=8, I=4, L=4, K=5, M=5, F=6, P=7, S=4,
                T=5, W=11, Y=7, V=4, B=4, Z=4, X=-1)
    diag["*"] = 1
    for c, v in diag.items():
        i = ALPHABET.index(c)
        assert BLOSUM62[i, i] == v, c
    assert BLOSUM62.max() == 11 and BLOSUM62.min() == -4


def test_blosum45_50_extrema():
    w = ALPHABET.index("W")
    assert BLOSUM45.max() == 15 and BLOSUM45[w, w] == 15 and BLOSUM45.min() == -5
    assert BLOSUM50.max() == 15 and BLOSUM50[w, w] == 15 and BLOSUM50.min() == -5


def test_blosum50_matches_durbin_fig2_2():
    cols = "HEAGW"
    with open(os.path.join(HERE, "golden", "durbin_fig2_5.txt")) as f:
        for line in f:
            t = line.split()
            if not t or t[0].startswith("#"):
                continue
            if t[0] == "row":
                r = ALPHABET.index(t[1])
                for c, v in zip(cols, t[2:]):
                    assert BLOSUM50[r, ALPHABET.index(c)] == int(v), (t[1], c)
            if t[0] == "diag":
                i = ALPHABET.index(t[1])
                assert BLOSUM50[i, i] == int(t[2])


def test_encode_roundtrip():
    s = "ARNDCQEGHILKMFPSTWYVBZX*"
    assert decode(encode(s)) == s
    assert decode(encode("uojb?")) == "XXXBX"
