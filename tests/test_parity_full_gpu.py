"""Full-size GPU parity ("next" item 1): the named configurations in full, in
the launch configuration bench.py times, element by element against the CPU oracle (bit-exact
int32, Eq.(1) of PAPER.md L12 §II; north_star "bit-exact per-sequence scores vs the CPU oracle
on all configs").

  * C3 in full (4,096 long sequences x the 5 queries, T = 3072: every pair takes the long path);
  * C2 in full (540k sequences) for queries 144 and 729 through the batch API with autotune;
  * a 1/8 round-robin shard of C2 (the per-GPU share of the 8-GPU C4 run) for query 5478 under
    the tuned configuration of the bench (menu 27: G = 32, R = 43, 4 strips) and with autotune;
  * every whole-warp (G = 32) configuration with queries of 2+ strips, so the multi-strip
    group stream (MULTI = true) runs in every instantiation, both regimes;
  * G-shard identity (SURVEY.md §8(c) pin 5, §8(e)): the round-robin shards of one database
    for G in {2, 4, 8}, each searched alone, reassembled by the gather's index map
    (dist.assemble), equal the G = 1 arrays and the oracle;
  * a 32-letter alphabet through both long-sequence paths (the pad letter is code 32).

The oracle runs on all host cores (OpenMP); each full-size case is ~20-30 s of oracle time on
the 16-core GPU host."""
import os

import numpy as np
import pytest
import torch

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from paper_conf_ipps_hainscobr11_b200 import dist as swdist
from workloads import gen
from workloads.matrices import BLOSUM62

pytestmark = pytest.mark.gpu


class _env:
    def __init__(self, **kv):
        self.kv = {k: str(v) for k, v in kv.items()}

    def __enter__(self):
        self.old = {k: os.environ.get(k) for k in self.kv}
        os.environ.update(self.kv)

    def __exit__(self, *a):
        for k, v in self.old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _check(got, ref, db, what):
    if not np.array_equal(got, ref):
        bad = np.nonzero(got != ref)[0]
        L = db.lengths
        raise AssertionError(f"{what}: {bad.size} mismatches: " +
                             ", ".join(f"#{i} len={L[i]} gpu={got[i]} oracle={ref[i]}" for i in bad[:10]))


def _batch(qs, W, db, T, env=None):
    with _env(**(env or {})):
        with swp.SmithWaterman(qs[0], W, 10, 2) as sw:
            sw.load_db(db.residues, db.offsets)
            out = sw.search_batch(qs, T)
            st = sw.stats()
    return out, st


def test_c3_full_parity():
    wl = gen.config("C3")
    db = wl.db
    assert db.num_seqs == 4096 and int(db.lengths.min()) >= 3073
    out, st = _batch(wl.queries, BLOSUM62, db, 3072)
    assert st["long_seqs"] == 4096 * len(wl.queries)
    for k, q in enumerate(wl.queries):
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
        _check(out[k], ref, db, f"C3 m={q.size}")


def test_c2_full_parity_144_729():
    wl = gen.config("C2")
    db = wl.db
    qs = [q for q in wl.queries if q.size in (144, 729)]
    out, st = _batch(qs, BLOSUM62, db, 3072)
    assert st["long_seqs"] == int((db.lengths >= 3072).sum()) * len(qs)
    for k, q in enumerate(qs):
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
        _check(out[k], ref, db, f"C2 m={q.size}")


def test_c2_shard8_5478_tuned_and_autotune():
    lens = gen.sp_lengths(540_000, seed=2)
    q = gen.make_query(5478)
    qs = [gen.make_query(L) for L in gen.C2_QUERY_LENGTHS]
    db = gen.build_database(lens, 2, qs, sel=gen.shard_indices(lens, 0, 8))
    ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
    out, _ = _batch([q], BLOSUM62, db, 3072, env={"SW_FORCE_MENU": 27})
    _check(out[0], ref, db, "C2/8 m=5478 menu 27")
    out, _ = _batch([q, q], BLOSUM62, db, 3072)   # autotune on (the first search of (5478, 3072))
    _check(out[0], ref, db, "C2/8 m=5478 autotune")
    _check(out[1], ref, db, "C2/8 m=5478 tuned")


def _g32_entries():
    import importlib.util
    path = os.path.join(os.path.dirname(swp.__file__), "csrc", "gen_menu.py")
    spec = importlib.util.spec_from_file_location("gen_menu", path)
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return [i for i, e in enumerate(mod.MENU) if e[0] == 0 and e[1] == 32]


@pytest.mark.parametrize("menu", _g32_entries())
def test_g32_multistrip_every_entry(menu):
    rng = np.random.default_rng(7000 + menu)
    lens = np.concatenate([np.arange(0, 30), rng.integers(30, 700, size=120), [1500, 3071, 3073, 5000]])
    rng.shuffle(lens)
    db = gen.build_database(lens.astype(np.int64), 70 + menu, None, alphabet_extra=True)
    for m in (1500, 3000, 5478):
        q = gen.make_query(m, seed=menu * 10 + m)
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
        for T, gs in ((1 << 30, "1"), (0, "1"), (1 << 30, "0")):
            try:
                with _env(SW_FORCE_MENU=menu, SW_GROUP_STREAM=gs):
                    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
                        sw.load_db(db.residues, db.offsets)
                        got = sw.search(T)
            except swp.SWError as e:
                assert e.status == swp.SW_E_UNSUPPORTED and "shared memory" in str(e)
                continue
            _check(got, ref, db, f"menu={menu} m={m} T={T} group_stream={gs}")


def test_gshard_identity():
    lens = gen.sp_lengths(20_000, seed=1)
    qs = [gen.make_query(L) for L in (144, 729, 5478)]
    full = gen.build_database(lens, 1, qs)
    g1, _ = _batch(qs, BLOSUM62, full, 3072)
    for k, q in enumerate(qs):
        _check(g1[k], oracle.scores(q, BLOSUM62, 10, 2, full.residues, full.offsets, threads=0), full,
               f"G=1 m={q.size}")
    n = lens.shape[0]
    for G in (2, 4, 8):
        n_pad = swdist.shard_size_bound(n, G)
        all_idx = torch.full((G, n_pad), -1, dtype=torch.int64)
        blocks = torch.zeros((G, len(qs), n_pad), dtype=torch.int32)
        for r in range(G):
            sel = swdist.shard_indices(lens, r, G)
            db = gen.build_database(lens, 1, qs, sel=sel)
            # the shard is bit-identical to the same sequences of the full database
            assert np.array_equal(db.residues, np.concatenate(
                [full.residues[full.offsets[i]:full.offsets[i + 1]] for i in sel]))
            out, _ = _batch(qs, BLOSUM62, db, 3072)
            all_idx[r, :sel.size] = torch.from_numpy(sel)
            blocks[r, :, :sel.size] = torch.from_numpy(out)
        got = swdist.assemble(all_idx, blocks, n).numpy()
        assert np.array_equal(got, g1), f"G={G}: {int((got != g1).sum())} scores differ from G=1"


@pytest.mark.parametrize("mode", ["t", "team"])
def test_alphabet_32_long_sequences(mode):
    """alphabet_size = 32 (the maximum): the database pad letter is code 32, one past the last
    real letter; the T-mode strip tables and the profile must give it its own column."""
    rng = np.random.default_rng(32)
    A = 32
    W = rng.integers(-5, 8, size=(A, A)).astype(np.int8)
    lens = np.concatenate([[5000, 3100, 4097, 513], rng.integers(0, 600, size=40)])
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    res = rng.integers(0, A, size=int(off[-1])).astype(np.uint8)
    res[: 4000] = 31          # runs of the last letter next to the pad
    db = gen.Database(res, off, np.arange(lens.size))
    for m in (100, 700, 3500):
        q = rng.integers(0, A, size=m).astype(np.uint8)
        q[:50] = 31
        ref = oracle.scores(q, W, 9, 1, db.residues, db.offsets, threads=0)
        for T in (0, 3000, 1 << 30):
            with _env(SW_LONG_MODE=mode):
                with swp.SmithWaterman(q, W, 9, 1) as sw:
                    sw.load_db(db.residues, db.offsets)
                    got = sw.search(T)
            _check(got, ref, db, f"A=32 mode={mode} m={m} T={T}")
