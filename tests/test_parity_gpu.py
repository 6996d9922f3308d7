"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element,
bit-exact int32 (north_star "bit-exact per-sequence scores vs the CPU oracle").

Inputs are seeded synthetic databases with the paper's workload shapes (workloads/gen.py).
Every compiled kernel configuration is exercised (SW_FORCE_MENU), both regimes (threshold
T = 0 sends everything to the intra-task/team path, T > max length everything to the
inter-task/group path), multi-strip queries, the 32-bit overflow recompute, ragged and
empty sequences."""
import os

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import ALPHABET, BLOSUM45, BLOSUM50, BLOSUM62

pytestmark = pytest.mark.gpu


def _db_from_lengths(lens, seed, extra=False, queries=None):
    return gen.build_database(np.asarray(lens, np.int64), seed, queries, alphabet_extra=extra)


def _gpu(query, W, rho, sigma, db, T, env=None):
    old = {}
    for k, v in (env or {}).items():
        old[k] = os.environ.get(k)
        os.environ[k] = str(v)
    try:
        with swp.SmithWaterman(query, W, rho, sigma) as sw:
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


def _oracle(query, W, rho, sigma, db):
    return oracle.scores(query, W, rho, sigma, db.residues, db.offsets, threads=0)


def _assert_equal(gpu, ref, db, what=""):
    if not np.array_equal(gpu, ref):
        bad = np.nonzero(gpu != ref)[0]
        L = db.lengths
        msg = ", ".join(f"#{i} len={L[i]} gpu={gpu[i]} oracle={ref[i]}" for i in bad[:10])
        raise AssertionError(f"{what}: {bad.size} mismatches: {msg}")


# ------------------------------------------------------------------ every configuration, both regimes
def _menu_entries():
    """s16x2 entries of csrc/gen_menu.py (the s32 recompute entry runs in team mode only)."""
    import importlib.util
    path = os.path.join(os.path.dirname(swp.__file__), "csrc", "gen_menu.py")
    spec = importlib.util.spec_from_file_location("gen_menu", path)
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return [i for i, e in enumerate(mod.MENU) if e[0] == 0]


MENU = _menu_entries()


@pytest.mark.parametrize("menu", MENU)
def test_every_config_both_regimes(menu):
    rng = np.random.default_rng(100 + menu)
    lens = np.concatenate([np.arange(0, 41), rng.integers(41, 700, size=300), [1500, 2047, 3071, 3072, 3073]])
    rng.shuffle(lens)
    db = _db_from_lengths(lens, seed=menu + 1, extra=True)
    for m in (1, 37, 144, 700):
        q = gen.make_query(m, seed=menu * 1000 + m)
        ref = _oracle(q, BLOSUM62, 10, 2, db)
        for T in (0, 1000, 1 << 30):
            try:
                out, st = _gpu(q, BLOSUM62, 10, 2, db, T, env={"SW_FORCE_MENU": menu})
            except swp.SWError as e:
                # a forced configuration whose profile replicas exceed shared memory is refused
                assert e.status == swp.SW_E_UNSUPPORTED and "shared memory" in str(e)
                continue
            _assert_equal(out, ref, db, f"menu={menu} m={m} T={T}")


@pytest.mark.parametrize("mode", ["team", "t8", "t2", "t1", "t2big2", "t1big4"])
@pytest.mark.parametrize("m", [1, 37, 144, 567, 1500])
def test_long_sequence_modes(mode, m):
    """Both long-sequence paths (team: strips of query rows; t: transposed, strips of the
    database sequence) on ragged long sequences, incl. the 35,213 maximum and lengths just
    around a strip multiple (512 positions per T-mode strip)."""
    rng = np.random.default_rng(77 + m)
    lens = np.concatenate([[35213, 512, 511, 513, 1024, 3072, 3073], rng.integers(3000, 12000, size=9),
                           rng.integers(0, 100, size=5)])
    db = _db_from_lengths(lens, seed=300 + m, extra=True)
    q = gen.make_query(m, seed=900 + m)
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    for T in (0, 3000):
        if mode == "team":
            env = {"SW_LONG_MODE": "team"}
        else:   # t<W>[big<S>]: phase-2 team size W, phase-1 (whole CTA) for pairs with >= S strips
            w, _, big = mode[1:].partition("big")
            env = {"SW_LONG_MODE": "t", "SW_T_TEAM": w, "SW_T_BIG": big or "1000000"}
        out, st = _gpu(q, BLOSUM62, 10, 2, db, T, env=env)
        _assert_equal(out, ref, db, f"mode={mode} m={m} T={T}")


@pytest.mark.parametrize("variant", ["share0", "share1", "chain0"])
@pytest.mark.parametrize("gang", ["2", "3", "8", "2:1", "5:3"])
@pytest.mark.parametrize("m", [1, 144, 1500])
def test_tmode_gangs(gang, m, variant):
    """T-mode gangs: the longest pairs spread over K CTAs (strip pipeline across CTAs through
    global row buffers and gpu-scope progress flags), SW_T_GANG = "K" (every long pair) or
    "K:items" (the items longest pairs); the other pairs take the CTA teams."""
    rng = np.random.default_rng(500 + m)
    lens = np.concatenate([[35213, 20000, 513, 512, 3073], rng.integers(3000, 15000, size=11),
                           rng.integers(0, 300, size=9)])
    db = _db_from_lengths(lens, seed=600 + m, extra=True)
    q = gen.make_query(m, seed=990 + m)
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    for T in (0, 3000):
        env = {"SW_LONG_MODE": "t", "SW_T_GANG": gang, "SW_T_GANG_SHARE": "1" if variant == "share1" else "0",
               "SW_T_GANG_CHAIN2": "0" if variant == "chain0" else "1"}
        out, _ = _gpu(q, BLOSUM62, 10, 2, db, T, env=env)
        _assert_equal(out, ref, db, f"gang={gang} m={m} T={T} {variant}")


def test_tmode_gangs_repeated_searches():
    """The gang hand-off words carry a per-launch epoch tag: repeated searches on one handle
    (the same buffers, the same strip indices) must never read a word of an earlier launch."""
    rng = np.random.default_rng(4)
    lens = np.concatenate([[35213, 30000, 20000], rng.integers(3000, 9000, size=6)])
    db = _db_from_lengths(lens, seed=61)
    os.environ.update({"SW_LONG_MODE": "t", "SW_T_GANG": "4"})
    try:
        for m in (144, 567):
            q = gen.make_query(m, seed=m + 1)
            ref = _oracle(q, BLOSUM62, 10, 2, db)
            with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
                sw.load_db(db.residues, db.offsets)
                for k in range(4):
                    _assert_equal(sw.search(0), ref, db, f"m={m} repeat {k}")
                outb = sw.search_batch([q, q, q], 0)
                for k in range(3):
                    _assert_equal(outb[k], ref, db, f"m={m} batch {k}")
    finally:
        os.environ.pop("SW_LONG_MODE", None)
        os.environ.pop("SW_T_GANG", None)


@pytest.mark.parametrize("team", [1, 2, 3, 5])
def test_team_mode_multi_warp(team):
    """Intra-task path with several warps chained over strips (progress-flag hand-off)."""
    rng = np.random.default_rng(7 + team)
    lens = np.concatenate([rng.integers(3000, 9000, size=12), rng.integers(0, 200, size=20)])
    db = _db_from_lengths(lens, seed=40 + team)
    q = gen.make_query(1500, seed=5 + team)
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    out, _ = _gpu(q, BLOSUM62, 10, 2, db, 0, env={"SW_FORCE_MENU": 8, "SW_FORCE_TEAM_WARPS": team,
                                                  "SW_LONG_MODE": "team"})
    _assert_equal(out, ref, db, f"team={team}")


# ------------------------------------------------------------------ thresholds / penalties / matrices
def test_threshold_invariance_c1_sample():
    wl = gen.config("C1", n_override=4000)
    q = wl.queries[0]
    db = wl.db
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    mx = int(db.lengths.max())
    for T in (0, 1, 2, 3071, 3072, 3073, mx, mx + 1, 36000):
        out, st = _gpu(q, BLOSUM62, 10, 2, db, T)
        _assert_equal(out, ref, db, f"T={T}")
        assert st["long_seqs"] == int((db.lengths >= T).sum())


@pytest.mark.parametrize("rho,sigma,W", [(12, 2, BLOSUM62), (10, 2, BLOSUM45), (3, 7, BLOSUM62), (0, 0, BLOSUM50),
                                         (1, 1, BLOSUM62), (116, 30, BLOSUM62)])
def test_penalties_and_matrices(rho, sigma, W):
    rng = np.random.default_rng(rho * 100 + sigma)
    lens = np.concatenate([rng.integers(0, 400, size=200), [3500, 4000]])
    db = _db_from_lengths(lens, seed=rho + 7 * sigma + 1, extra=True)
    for m in (60, 513):
        q = gen.make_query(m, seed=m + rho)
        ref = _oracle(q, W, rho, sigma, db)
        for T in (0, 3072):
            out, _ = _gpu(q, W, rho, sigma, db, T)
            _assert_equal(out, ref, db, f"rho={rho} sigma={sigma} m={m} T={T}")


def test_asymmetric_random_matrix():
    rng = np.random.default_rng(5)
    A = 24
    W = rng.integers(-6, 9, size=(A, A)).astype(np.int8)
    db = _db_from_lengths(rng.integers(0, 300, size=150), seed=9, extra=True)
    q = rng.integers(0, A, size=200).astype(np.uint8)
    ref = _oracle(q, W, 7, 1, db)
    for T in (0, 150, 1 << 20):
        out, _ = _gpu(q, W, 7, 1, db, T)
        _assert_equal(out, ref, db, f"asym T={T}")


def test_small_alphabet_dna_like():
    rng = np.random.default_rng(6)
    W = np.array([[5, -4, -4, -4], [-4, 5, -4, -4], [-4, -4, 5, -4], [-4, -4, -4, 5]], np.int8)
    lens = rng.integers(0, 1000, size=100)
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    res = rng.integers(0, 4, size=int(off[-1])).astype(np.uint8)
    db = gen.Database(res, off, np.arange(100))
    q = rng.integers(0, 4, size=333).astype(np.uint8)
    ref = _oracle(q, W, 10, 1, db)
    for T in (0, 500, 5000):
        out, _ = _gpu(q, W, 10, 1, db, T)
        _assert_equal(out, ref, db, f"dna T={T}")


# ------------------------------------------------------------------ long queries / long sequences
def test_long_query_5478_vs_long_db():
    lens = gen.long_lengths(24, seed=3, max_len=12000)
    q = gen.make_query(5478)
    db = gen.build_database(lens, 3, [q])
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    for T in (0, 1 << 30):
        out, _ = _gpu(q, BLOSUM62, 10, 2, db, T)
        _assert_equal(out, ref, db, f"5478 T={T}")


# ------------------------------------------------------------------ overflow recompute (16 -> 32 bit)
def test_overflow_recompute_homopolymers():
    w = ALPHABET.index("W")
    lens = [3100, 2900, 3000, 2978, 2979, 100, 0, 5]
    res = np.concatenate([np.full(n, w, np.uint8) for n in lens])
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    db = gen.Database(res, off, np.arange(len(lens)))
    q = np.full(3050, w, np.uint8)
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    assert ref[0] == 3050 * 11 and ref[0] > 32767
    for T in (0, 1 << 30):
        out, st = _gpu(q, BLOSUM62, 10, 2, db, T)
        _assert_equal(out, ref, db, f"homopolymer T={T}")
        assert st["recomputed_s32"] > 0


def test_overflow_planted_self_copy_blosum45():
    q = gen.make_query(5478)
    rng = np.random.default_rng(11)
    other = [rng.integers(0, 20, size=int(n)).astype(np.uint8) for n in rng.integers(10, 2000, size=40)]
    seqs = other[:20] + [q.copy()] + other[20:] + [np.concatenate([q[:3000], q[:3000]])]
    off = np.concatenate([[0], np.cumsum([s.size for s in seqs])]).astype(np.int64)
    db = gen.Database(np.concatenate(seqs), off, np.arange(len(seqs)))
    ref = _oracle(q, BLOSUM45, 10, 2, db)
    assert ref.max() > 32767
    for T in (0, 3072, 1 << 30):
        out, st = _gpu(q, BLOSUM45, 10, 2, db, T)
        _assert_equal(out, ref, db, f"self-copy T={T}")
        assert st["recomputed_s32"] >= 1


def test_no_recompute_on_random_db():
    wl = gen.config("C1", n_override=2000)
    out, st = _gpu(wl.queries[0], BLOSUM62, 10, 2, wl.db, 3072)
    assert st["recomputed_s32"] == 0


# ------------------------------------------------------------------ layout / order / batch
def test_permutation_only_permutes_output():
    rng = np.random.default_rng(21)
    lens = rng.integers(0, 800, size=500)
    db = _db_from_lengths(lens, seed=21)
    q = gen.make_query(300)
    out1, _ = _gpu(q, BLOSUM62, 10, 2, db, 500)
    perm = rng.permutation(500)
    seqs = [db.residues[db.offsets[i]:db.offsets[i + 1]] for i in perm]
    off = np.concatenate([[0], np.cumsum([s.size for s in seqs])]).astype(np.int64)
    db2 = gen.Database(np.concatenate(seqs), off, perm)
    out2, _ = _gpu(q, BLOSUM62, 10, 2, db2, 500)
    assert np.array_equal(out2, out1[perm])


def test_batch_equals_single_queries():
    wl = gen.config("C1", n_override=3000)
    qs = [gen.make_query(L) for L in (144, 375, 729, 1500, 5478, 37)]
    with swp.SmithWaterman(qs[0], BLOSUM62, 10, 2) as sw:
        sw.load_db(wl.db.residues, wl.db.offsets)
        outb = sw.search_batch(qs, 3072)
        for k, q in enumerate(qs):
            sw.set_query(q)
            assert np.array_equal(sw.search(3072), outb[k])
    for k in (0, 5):
        _assert_equal(outb[k], _oracle(qs[k], BLOSUM62, 10, 2, wl.db), wl.db, f"batch q{k}")


def test_empty_and_degenerate():
    q = gen.make_query(20)
    # empty database
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(np.zeros(0, np.uint8), np.zeros(1, np.int64))
        assert sw.search(3072).shape == (0,)
    # all-empty sequences and one residue
    db = gen.Database(np.array([3], np.uint8), np.array([0, 0, 0, 1, 1], np.int64), np.arange(4))
    out, _ = _gpu(q, BLOSUM62, 10, 2, db, 0)
    assert np.array_equal(out, _oracle(q, BLOSUM62, 10, 2, db))
    # all-negative matrix: every score 0
    Wn = np.full((24, 24), -2, np.int8)
    db = _db_from_lengths([5, 50, 500, 5000], seed=3)
    out, _ = _gpu(q, Wn, 0, 0, db, 100)
    assert not out.any()


# ------------------------------------------------------------------ full C1 (BASELINE config 1) and sampled C2
def test_c1_full_parity():
    wl = gen.config("C1")
    q = wl.queries[0]
    ref = _oracle(q, BLOSUM62, 10, 2, wl.db)
    out, st = _gpu(q, BLOSUM62, 10, 2, wl.db, 3072)
    _assert_equal(out, ref, wl.db, "C1")
    assert st["long_seqs"] == int((wl.db.lengths >= 3072).sum())


def test_c2_full_size_sampled():
    """Full C2 database (540k seqs) in the bench's launch configuration; the oracle checks a
    deterministic sample (the 64 longest + every 5000th sequence) for each query."""
    wl = gen.config("C2")
    db = wl.db
    L = db.lengths
    order = np.argsort(-L, kind="stable")
    sample = np.unique(np.concatenate([order[:64], np.arange(0, db.num_seqs, 5000)]))
    sub_lens = L[sample]
    sub_off = np.concatenate([[0], np.cumsum(sub_lens)]).astype(np.int64)
    sub_res = np.concatenate([db.residues[db.offsets[i]:db.offsets[i + 1]] for i in sample])
    with swp.SmithWaterman(wl.queries[0], BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        outb = sw.search_batch(wl.queries, 3072)
    for k, q in enumerate(wl.queries):
        ref = oracle.scores(q, BLOSUM62, 10, 2, sub_res, sub_off, threads=0)
        got = outb[k][sample]
        assert np.array_equal(got, ref), (k, np.nonzero(got != ref)[0][:10])
        assert (outb[k] >= 0).all()


# ------------------------------------------------------------------ automatic threshold (f1)
@pytest.mark.parametrize("cfg", ["C1", "C3"])
def test_auto_threshold_parity(cfg):
    if cfg == "C1":
        wl = gen.config("C1", n_override=3000)
        db, q = wl.db, wl.queries[0]
    else:
        lens = gen.long_lengths(64, seed=3, max_len=9000)
        q = gen.make_query(567)
        db = gen.build_database(lens, 3, [q])
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        out = sw.search(swp.SW_AUTO_THRESHOLD)
        T = sw.last_threshold()
    _assert_equal(out, ref, db, f"auto T={T}")
    assert T >= 0


# ------------------------------------------------------------------ C5 recipe (TrEMBL-scale config)
def test_c5_slice_blosum45_parity():
    """A 1/20000 round-robin slice of C5 (50M sequences, mean length 320, BLOSUM45 10/2, the
    benchmark query lengths): full parity against the oracle for three of the 20 queries."""
    full = gen.sp_lengths(50_000_000, seed=5, mu=5.4270)
    order = np.argsort(-full, kind="stable")
    view = np.sort(order[::20000])
    lens = full[view]
    qs = [gen.make_query(L) for L in gen.BENCH_QUERY_LENGTHS]
    db = gen.build_database(lens, 5, qs)
    assert db.num_seqs == 2500 and lens.max() == full.max()
    for m in (144, 1000, 5478):
        q = gen.make_query(m)
        ref = _oracle(q, BLOSUM45, 10, 2, db)
        out, _ = _gpu(q, BLOSUM45, 10, 2, db, 3072)
        _assert_equal(out, ref, db, f"C5 slice m={m}")


# ------------------------------------------------------------------ north-star invariant and maximum sizes
def test_query_subject_swap_symmetry():
    """north_star: "scores are unchanged when query and subject are swapped under a symmetric
    matrix" (Eq.(1) with w symmetric is symmetric in (q, d): transpose the DP grid, E <-> F).
    Each database sequence becomes the query of its own search against a one-sequence
    database holding the original query; both directions go through the CUDA path (group and
    long regimes) and both equal the oracle."""
    q = gen.make_query(375)
    lens = [1, 2, 17, 144, 375, 376, 1500, 3100, 5478]
    db = _db_from_lengths(lens, seed=41, queries=[q])
    fwd, _ = _gpu(q, BLOSUM62, 10, 2, db, 1000)
    _assert_equal(fwd, _oracle(q, BLOSUM62, 10, 2, db), db, "forward")
    one = gen.Database(q.copy(), np.array([0, q.size], np.int64), np.arange(1))
    for k in range(db.num_seqs):
        d = db.residues[db.offsets[k]:db.offsets[k + 1]]
        for T in (0, 1 << 20):
            rev, _ = _gpu(d, BLOSUM62, 10, 2, one, T)
            assert rev[0] == fwd[k], f"seq {k} (len {d.size}) T={T}: swapped {rev[0]} != {fwd[k]}"


def test_maximum_query_and_sequence_lengths():
    """The limits include/sw.h declares: a query of SW_MAX_QUERY_LEN = 65536 residues over a
    2-letter alphabet (its profile fits SW_MAX_PROFILE_BYTES; many strips; one sequence holds
    an 8000-residue copy of it, so the s16 pass saturates and the 32-bit recompute decides),
    protein queries of 8192 (profile in shared memory) and 65536 (long-query mode), and a
    database sequence of SW_MAX_SEQ_LEN = 1,048,512 residues in both regimes."""
    W2 = np.array([[5, -4], [-4, 5]], np.int8)
    q = (gen.u01(1007, "query", np.arange(1 << 16, dtype=np.uint64)) < 0.5).astype(np.uint8)
    parts = [(gen.u01(1043 + k, "res", np.arange(n, dtype=np.uint64)) < 0.5).astype(np.uint8)
             for k, n in enumerate([1, 31, 500, 3100])] + [q[1000:9000]]
    offs = np.concatenate([[0], np.cumsum([x.size for x in parts])]).astype(np.int64)
    db = gen.Database(np.concatenate(parts).astype(np.uint8), offs, np.arange(len(parts)))
    ref = _oracle(q, W2, 10, 2, db)
    assert ref[-1] == 5 * 8000
    for T in (0, 3072):
        out, st = _gpu(q, W2, 10, 2, db, T)
        _assert_equal(out, ref, db, f"query 65536 (2 letters) T={T}")
        assert st["recomputed_s32"] >= 1

    q = gen.make_query(8192, seed=9)
    db = _db_from_lengths([1, 31, 500, 3100, 9000], seed=45, queries=[q])
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    for T in (0, 3072):
        out, _ = _gpu(q, BLOSUM62, 10, 2, db, T)
        _assert_equal(out, ref, db, f"protein query 8192 T={T}")
    # a protein query of SW_MAX_QUERY_LEN residues: its profile exceeds shared memory, so the
    # search runs in long-query mode (T-mode for every pair, tests/test_long_query_gpu.py)
    q = gen.make_query(1 << 16, seed=7)
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    out, st = _gpu(q, BLOSUM62, 10, 2, db, 3072)
    _assert_equal(out, ref, db, "protein query 65536")
    assert st["long_seqs"] == db.num_seqs

    q = gen.make_query(144)
    lmax = (1 << 20) - 64
    db = _db_from_lengths([lmax, 7, 3073], seed=44)
    assert db.lengths.max() == lmax
    ref = _oracle(q, BLOSUM62, 10, 2, db)
    for T in (0, 1 << 20):
        out, _ = _gpu(q, BLOSUM62, 10, 2, db, T)
        _assert_equal(out, ref, db, f"max sequence T={T}")
