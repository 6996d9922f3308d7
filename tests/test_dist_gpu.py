"""The multi-GPU code path on the GPU: an NCCL process group (one rank, the
pool gives one GPU), the shard padded for the uniform gather, the library writing straight into
the gather's send block, one NCCL all_gather_into_tensor and the index map back to global order
— bit-exact against the oracle.  World sizes 2 and 3 of the same host logic run on CPU with
gloo (tests/test_dist_gloo.py)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(port, errq):
    try:
        import torch
        import torch.distributed as dist

        import oracle
        import paper_conf_ipps_hainscobr11_b200 as swp
        from paper_conf_ipps_hainscobr11_b200.dist import ScoreGather, shard_indices
        from workloads import gen
        from workloads.matrices import BLOSUM62

        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dev = torch.device("cuda", 0)
        torch.cuda.set_device(dev)
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
        qs = [gen.make_query(144, seed=1), gen.make_query(1500, seed=2)]
        lens = np.concatenate([gen.sp_lengths(6000, seed=11), [3500, 9000]])
        sel = shard_indices(lens, 0, 1)
        db = gen.build_database(lens, 11, qs, sel=sel)
        g = ScoreGather(db.global_index, lens.shape[0], len(qs), device=dev)
        with swp.SmithWaterman(qs[0], BLOSUM62, 10, 2) as sw:
            sw.load_db(db.residues, ScoreGather.pad_offsets(db.offsets, g.n_pad))
            stream = torch.cuda.current_stream(dev)
            sw.search_batch_into(qs, g.send_ptr(), 3072, stream.cuda_stream)
            g.gather()
            out = g.to_global().cpu().numpy()
        for k, q in enumerate(qs):
            ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets, threads=0)
            bad = np.nonzero(out[k] != ref)[0]
            assert bad.size == 0, f"query {k}: {bad.size} mismatches, first {bad[:5]}"
        dist.destroy_process_group()
    except Exception as e:  # reported to the parent
        errq.put(f"{type(e).__name__}: {e}")


def test_nccl_score_gather_world1():
    ctx = mp.get_context("spawn")
    errq = ctx.SimpleQueue()
    p = ctx.Process(target=_worker, args=(_free_port(), errq))
    p.start()
    p.join(timeout=300)
    errs = []
    while not errq.empty():
        errs.append(errq.get())
    assert not errs, errs
    assert p.exitcode == 0
