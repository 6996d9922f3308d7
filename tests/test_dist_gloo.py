"""Multi-process (world_size 2 and 3, gloo on CPU) test of the multi-GPU path's host logic:
round-robin sharding over the length-sorted order and the final score gather back into the
caller's database order.  The GPU search itself is replaced by a
deterministic per-sequence function; the collective and index plumbing are the real ones."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_ipps_hainscobr11_b200 import dist as swdist
from workloads import gen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def fake_scores(q, gidx):
    return ((gidx * 7919 + q * 104729) % 100003).astype(np.int32)


def _worker(rank, world, port, n_total, nq, errq, all_gather=False):
    import torch
    import torch.distributed as dist
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        lens = gen.sp_lengths(n_total, seed=9)
        sel = swdist.shard_indices(lens, rank, world)
        g = swdist.ScoreGather(sel, n_total, nq, all_gather=all_gather)
        # the "search" writes [nq, n_pad] contiguous (shard padded with empty sequences -> 0)
        for q in range(nq):
            g.send[q, : sel.shape[0]] = torch.from_numpy(fake_scores(q, sel))
            g.send[q, sel.shape[0]:] = 0
        g.gather()
        if all_gather or rank == 0:
            out = g.to_global().numpy()
            want = np.stack([fake_scores(q, np.arange(n_total)) for q in range(nq)])
            assert np.array_equal(out, want)
        else:
            assert g.recv is None   # gather to rank 0: no receive buffer elsewhere
        # balance: residues per shard within one max length of each other
        tot = torch.tensor([int(lens[sel].sum())], dtype=torch.int64)
        allt = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allt, tot)
        vals = [int(t.item()) for t in allt]
        assert max(vals) - min(vals) <= int(lens.max())
        assert sum(vals) == int(lens.sum())
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - reported to the parent
        errq.put(f"rank {rank}: {type(e).__name__}: {e}")


@pytest.mark.parametrize("all_gather", [False, True])
@pytest.mark.parametrize("world", [2, 3])
def test_shard_and_gather_gloo(world, all_gather):
    ctx = mp.get_context("spawn")
    errq = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 10007, 3, errq, all_gather)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=120)
    errs = []
    while not errq.empty():
        errs.append(errq.get())
    assert not errs, errs
    assert all(p.exitcode == 0 for p in procs)


def test_shard_rule_matches_generator():
    lens = gen.sp_lengths(5000, seed=4)
    for world in (1, 2, 4, 8):
        for r in range(world):
            assert np.array_equal(swdist.shard_indices(lens, r, world), gen.shard_indices(lens, r, world))


def test_pad_offsets():
    off = np.array([0, 3, 3, 10], np.int64)
    p = swdist.ScoreGather.pad_offsets(off, 6)
    assert p.tolist() == [0, 3, 3, 10, 10, 10, 10]


def _c4_worker(rank, world, port, errq):
    """bench.py's C4 path (C2's database split over the ranks, strong scaling) with a stub
    search: every rank builds only its shard, writes its [nq, n_pad] block, one gather to rank
    0, rank 0 reassembles the global order and checks it against the stub over the full DB."""
    import torch
    import torch.distributed as dist
    try:
        import bench
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        qs, db, lens_all, *_ = bench.make_workload("C4", rank, world, n_override=6000)
        n_total = int(lens_all.shape[0])
        assert n_total == 6000 and bench.SCALING["C4"] == "strong"
        assert np.array_equal(db.global_index, gen.shard_indices(lens_all, rank, world))
        g = swdist.ScoreGather(db.global_index, n_total, len(qs))
        padded = swdist.ScoreGather.pad_offsets(db.offsets, g.n_pad)
        assert padded.shape[0] - 1 == g.n_pad and padded[-1] == db.total_residues
        for q in range(len(qs)):
            g.send[q, : db.num_seqs] = torch.from_numpy(fake_scores(q, db.global_index))
        g.gather()
        if rank == 0:
            out = g.to_global().numpy()
            want = np.stack([fake_scores(q, np.arange(n_total)) for q in range(len(qs))])
            assert np.array_equal(out, want)
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        errq.put(f"rank {rank}: {type(e).__name__}: {e}")


@pytest.mark.parametrize("world", [2, 3])
def test_c4_strong_scaling_path_gloo(world):
    ctx = mp.get_context("spawn")
    errq = ctx.SimpleQueue()
    port = _free_port()
    procs = [ctx.Process(target=_c4_worker, args=(r, world, port, errq)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=180)
    errs = []
    while not errq.empty():
        errs.append(errq.get())
    assert not errs, errs
    assert all(p.exitcode == 0 for p in procs)
