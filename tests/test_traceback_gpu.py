"""Device traceback (sw_align): the returned alignment is a valid local
alignment whose own score — recomputed here from its runs, independently of Eq.(1) — equals
the oracle's optimal score; Durbin et al. Fig.2.5's alignment is reproduced."""
import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM45, BLOSUM50, BLOSUM62, encode

pytestmark = pytest.mark.gpu


def score_runs(q, d, W, rho, sigma, al):
    """Score of an alignment given as runs: sum of w over M columns, rho + (len-1)*sigma per
    gap run; also checks that the runs consume exactly q[q_begin:q_end] and d[d_begin:d_end]."""
    i, j, s = al["q_begin"], al["d_begin"], 0
    for op, n in al["runs"]:
        assert n >= 1
        if op == "M":
            for _ in range(n):
                s += int(W[q[i]][d[j]])
                i += 1
                j += 1
        elif op == "I":
            s -= rho + (n - 1) * sigma
            j += n
        else:
            s -= rho + (n - 1) * sigma
            i += n
    assert (i, j) == (al["q_end"], al["d_end"])
    return s


def test_durbin_fig2_5_alignment():
    q, d = encode("HEAGAWGHEE"), encode("PAWHEAE")
    with swp.SmithWaterman(q, BLOSUM50, 8, 8) as sw:
        sw.load_db(d, np.array([0, d.size], np.int64))
        al = sw.align(0)
    assert al["score"] == 28
    assert score_runs(q, d, BLOSUM50, 8, 8, al) == 28
    assert (al["q_begin"], al["q_end"], al["d_begin"], al["d_end"]) == (4, 9, 1, 5)
    assert al["cigar"] == "2M1D2M"        # AWGHE / AW-HE


@pytest.mark.parametrize("rho,sigma,W", [(10, 2, BLOSUM62), (12, 2, BLOSUM45), (3, 7, BLOSUM62), (0, 0, BLOSUM62)])
def test_random_alignments_score_optimal(rho, sigma, W):
    rng = np.random.default_rng(rho * 31 + sigma)
    q = gen.make_query(300, seed=rho + 1)
    seqs = [rng.integers(0, 20, size=int(n)).astype(np.uint8) for n in rng.integers(0, 500, size=12)]
    seqs.append(np.concatenate([seqs[0][:50], q[40:200], seqs[1][:30]]))       # planted homologue
    mut = q[100:260].copy()
    mut[::7] = rng.integers(0, 20, size=mut[::7].size)
    seqs.append(np.concatenate([mut[:60], mut[75:]]))                           # with a deletion
    off = np.concatenate([[0], np.cumsum([s.size for s in seqs])]).astype(np.int64)
    res = np.concatenate(seqs)
    ref = oracle.scores(q, W, rho, sigma, res, off)
    with swp.SmithWaterman(q, W, rho, sigma) as sw:
        sw.load_db(res, off)
        for k, s in enumerate(seqs):
            al = sw.align(k)
            assert al["score"] == ref[k], (k, al["score"], ref[k])
            if ref[k] == 0:
                assert al["runs"] == []
                continue
            assert score_runs(q, s, W, rho, sigma, al) == ref[k]
            assert 0 <= al["q_begin"] < al["q_end"] <= q.size and 0 <= al["d_begin"] < al["d_end"] <= s.size


def test_traceback_long_pair():
    q = gen.make_query(1500)
    d = np.concatenate([gen.make_query(4000, seed=5), q[200:1300], gen.make_query(3000, seed=6)])
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(d, np.array([0, d.size], np.int64))
        al = sw.align(0)
    ref = oracle.pair(q, d, BLOSUM62, 10, 2)
    assert al["score"] == ref
    assert score_runs(q, d, BLOSUM62, 10, 2, al) == ref
    assert al["d_begin"] <= 4000 + 10 and al["d_end"] >= 4000 + 1090


def test_align_errors():
    with swp.SmithWaterman(gen.make_query(10), BLOSUM62, 10, 2) as sw:
        with pytest.raises(swp.SWError) as e:
            sw.align(0)
        assert e.value.status == swp.SW_E_STATE
        sw.load_db(np.zeros(0, np.uint8), np.array([0, 0], np.int64))
        al = sw.align(0)                          # empty sequence
        assert al["score"] == 0 and al["runs"] == []
        with pytest.raises(swp.SWError) as e:
            sw.align(5)
        assert e.value.status == swp.SW_E_INVALID


def test_local_hit_in_long_sequence_bounded_box():
    """A planted homologous window inside a 30,000-residue sequence: the bounded-memory traceback
    (score + end cell, anchored reverse sweep for the start, directions for the bounding box only)
    returns an optimal alignment inside the window's neighbourhood, rescored independently."""
    rng = np.random.default_rng(21)
    q = gen.make_query(300, seed=5)
    d = rng.integers(0, 20, size=30000).astype(np.uint8)
    win = q[40:260].copy()
    mut = rng.random(win.size) < 0.25
    win[mut] = rng.integers(0, 20, size=int(mut.sum()))
    d[17000:17000 + win.size] = win
    off = np.array([0, d.size], np.int64)
    ref = oracle.scores(q, BLOSUM62, 10, 2, d, off)
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(d, off)
        al = sw.align(0)
    assert al["score"] == ref[0]
    assert score_runs(q, d, BLOSUM62, 10, 2, al) == ref[0]
    assert 16000 < al["d_begin"] < al["d_end"] < 18000


def test_top_hits_match_numpy_order():
    """sw_top_hits: the k largest scores (ties by the smaller index), best first, against a
    numpy lexsort of the same array — real search output with many ties, negative and large
    values, k beyond n."""
    wl = gen.config("C1", n_override=20000)
    q = wl.queries[0]
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(wl.db.residues, wl.db.offsets)
        out = sw.search(3072)
        cases = [out, np.array([5, -3, 7, 7, 2**31 - 1, -2**31, 0, 7], np.int32),
                 np.random.default_rng(3).integers(-5, 5, size=100000).astype(np.int32)]
        for arr in cases:
            order = np.lexsort((np.arange(arr.size), -arr.astype(np.int64)))
            for k in (1, 10, 1000, arr.size, arr.size + 5):
                idx, val = sw.top_hits(arr, k)
                kk = min(k, arr.size)
                assert np.array_equal(idx, order[:kk]), (k, idx[:10], order[:10])
                assert np.array_equal(val, arr[order[:kk]])
        idx, val = sw.top_hits(out, 0)
        assert idx.size == 0
        # the top hits' alignments rescore to their search scores
        idx, val = sw.top_hits(out, 5)
        for i, v in zip(idx, val):
            al = sw.align(int(i))
            assert al["score"] == v
            s, e = wl.db.offsets[i], wl.db.offsets[i + 1]
            assert score_runs(q, wl.db.residues[s:e], BLOSUM62, 10, 2, al) == v
