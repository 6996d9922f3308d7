"""Input generator: determinism and shard invariance."""
import numpy as np

from workloads import gen


def test_deterministic_and_shard_invariant():
    lens = gen.sp_lengths(3000, seed=11)
    qs = [gen.make_query(50), gen.make_query(80)]
    full = gen.build_database(lens, 11, qs)
    full2 = gen.build_database(lens, 11, qs)
    assert np.array_equal(full.residues, full2.residues)
    for world in (2, 3, 4):
        seen = 0
        for r in range(world):
            sel = gen.shard_indices(lens, r, world)
            sh = gen.build_database(lens, 11, qs, sel=sel)
            for k, g in enumerate(sh.global_index):
                a = sh.residues[sh.offsets[k]:sh.offsets[k + 1]]
                b = full.residues[full.offsets[g]:full.offsets[g + 1]]
                assert np.array_equal(a, b)
            seen += sh.num_seqs
        assert seen == 3000


def test_round_robin_balances_residues():
    lens = gen.sp_lengths(20000, seed=1)
    tot = [int(lens[gen.shard_indices(lens, r, 8)].sum()) for r in range(8)]
    assert max(tot) - min(tot) <= int(lens.max())


def test_sp_length_model_shape():
    lens = gen.sp_lengths(200000, seed=2)
    assert lens.max() == gen.MAX_LEN and lens.min() >= 2
    assert 340 < lens.mean() < 365
    frac_long = (lens >= 3072).mean()
    assert 0.0008 < frac_long < 0.0020       # ~0.12% over the default threshold


def test_long_lengths():
    lens = gen.long_lengths(512, seed=3)
    assert lens.min() >= 3073 and lens.max() == gen.MAX_LEN


def test_residue_codes_and_queries():
    q = gen.make_query(144)
    assert q.shape == (144,) and q.max() < 20
    assert np.array_equal(q, gen.make_query(144))
    db = gen.build_database(gen.sp_lengths(500, 5), 5, alphabet_extra=True)
    assert db.residues.max() <= 23
