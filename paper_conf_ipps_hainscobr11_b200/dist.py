"""Multi-GPU partitioning and the final score gather.

The search shards naturally: every (query, database sequence) score is independent
("kernel tasks are independent ... the running time will scale almost linearly with the
number of GPUs", §IV-B; "pleasantly parallel", L28 §V).  One process per GPU
loads a shard of the database and searches it with the C ABI; the only collective is one
gather of the int32 scores to rank 0 (NCCL over NVLink on the B200 box, gloo in the CPU tests).

Partition rule: stable sort of all lengths descending, rank r takes sorted positions
r, r + G, r + 2G, ... (round-robin).  Every shard then has the same length profile, so both
regimes (short / long, for any threshold) are balanced to within one sequence per rank.
"""
from __future__ import annotations

import numpy as np


def shard_indices(lengths_all, rank: int, world: int) -> np.ndarray:
    """Global indices of rank's shard (increasing order)."""
    lengths_all = np.asarray(lengths_all)
    if world == 1:
        return np.arange(lengths_all.shape[0], dtype=np.int64)
    order = np.argsort(-lengths_all, kind="stable")
    return np.sort(order[rank::world]).astype(np.int64)


def shard_size_bound(n_total: int, world: int) -> int:
    """Uniform per-rank row count for the gather (ceil(N / world))."""
    return -(-n_total // world)


def assemble(all_idx, blocks, n_total: int):
    """Scores in global database order from per-rank blocks.

    all_idx: [world, n_pad] global index of every row of every rank's block (-1 = padding);
    blocks:  [world, nq, n_pad] the ranks' score blocks.  Returns [nq, n_total] (torch)."""
    import torch
    world, nq = blocks.shape[0], blocks.shape[1]
    out = torch.empty((nq, int(n_total)), dtype=blocks.dtype, device=blocks.device)
    for r in range(world):
        v = all_idx[r] >= 0
        out[:, all_idx[r][v]] = blocks[r][:, v]
    return out


class ScoreGather:
    """Gathers per-rank score blocks [nq, n_local] into [nq, n_total] in global order.

    The index map is exchanged once at construction (not on the timed path); each search then
    costs one collective of nq * ceil(N / world) int32 per rank: a gather to rank 0 (default;
    only rank 0 holds the world * nq * n_pad receive buffer, 4 GB for C5 with 20 queries) or,
    with all_gather=True, an all_gather_into_tensor that lands every score on every rank."""

    def __init__(self, global_index, n_total: int, nq: int, group=None, device=None, all_gather: bool = False):
        import torch
        import torch.distributed as dist

        self.dist = dist
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.all_gather = bool(all_gather)
        self.n_total = int(n_total)
        self.nq = int(nq)
        self.n_pad = shard_size_bound(self.n_total, self.world)
        gi = np.asarray(global_index, dtype=np.int64)
        self.n_local = int(gi.shape[0])
        if self.n_local > self.n_pad:
            raise ValueError("shard larger than ceil(N / world)")
        dev = device if device is not None else torch.device("cpu")
        idx = torch.full((self.n_pad,), -1, dtype=torch.int64, device=dev)
        idx[: self.n_local] = torch.from_numpy(gi).to(dev)
        flat = torch.empty((self.world * self.n_pad,), dtype=torch.int64, device=dev)
        dist.all_gather_into_tensor(flat, idx, group=group)   # flat output: gloo and NCCL
        all_idx = flat.view(self.world, self.n_pad)
        self.all_idx = all_idx
        self.send = torch.zeros((self.nq, self.n_pad), dtype=torch.int32, device=dev)
        self.holds_all = self.all_gather or self.rank == 0
        if self.holds_all:
            self.recv_flat = torch.empty((self.world * self.nq * self.n_pad,), dtype=torch.int32, device=dev)
            self.recv = self.recv_flat.view(self.world, self.nq, self.n_pad)
        else:
            self.recv_flat = self.recv = None

    def send_ptr(self) -> int:
        """Device pointer of the [nq, n_pad] block the search writes into.  The caller loads
        its shard padded with empty sequences up to n_pad (they score 0 and are dropped by the
        index map), so the library's contiguous [nq, n_pad] output is exactly this block."""
        return self.send.data_ptr()

    @staticmethod
    def pad_offsets(offsets, n_pad: int):
        """CSR offsets of a shard extended with empty sequences up to n_pad."""
        off = np.asarray(offsets, dtype=np.int64)
        extra = n_pad - (off.shape[0] - 1)
        if extra < 0:
            raise ValueError("shard larger than n_pad")
        return np.concatenate([off, np.full(extra, off[-1], dtype=np.int64)])

    def gather(self):
        """Collective: every rank calls it; returns nothing (the data lands in self.recv on
        rank 0, or on every rank with all_gather=True)."""
        if self.all_gather:
            self.dist.all_gather_into_tensor(self.recv_flat, self.send.view(-1), group=self.group)
        else:
            dst = self.dist.get_global_rank(self.group, 0) if self.group is not None else 0
            glist = list(self.recv.unbind(0)) if self.rank == 0 else None
            self.dist.gather(self.send, gather_list=glist, dst=dst, group=self.group)

    def to_global(self):
        """[nq, n_total] scores in global database order (after gather(); rank 0, or every
        rank with all_gather=True)."""
        if not self.holds_all:
            raise RuntimeError("to_global() is valid on rank 0 only (gather to rank 0)")
        return assemble(self.all_idx, self.recv, self.n_total)
