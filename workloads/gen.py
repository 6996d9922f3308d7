"""Seeded, shard-invariant synthetic workloads (SURVEY.md §8(d) "Synthetic workloads").

This module produces INPUTS only — database lengths/residues and queries — and holds none
of the method's arithmetic.  Both the oracle (tests, cpu_baseline) and the CUDA path
(bench, tests) consume what it returns; neither side imports the other.

Randomness is counter-based (splitmix64 of (seed, stream, index)), so any shard of a
database can be generated on its own and is bit-identical to the same sequences of the
full database.

Recipe (DESIGN.md "Input recipe" restates it):
  * Swiss-Prot-shaped lengths ("resembles a log-normal distribution", §II-C):
    n = clamp(round(exp(mu + s*Z)), 2, 35213), mu = 5.5219, s = 0.8262 (reading c14);
    a fraction 1e-4 re-drawn log-uniform in [10000, 35213]; the longest set to 35213.
  * residues i.i.d. from Robinson-Robinson background frequencies over the 20 standard
    amino acids (codes 0..19 of ARNDCQEGHILKMFPSTWYV);
  * planted hits: a fraction 1e-4 (at least 4) of sequences carry a window of one of the
    configured queries with 30% substitutions and 2% indels, inside their own length slot
    (lengths/offsets never depend on the queries);
  * queries: i.i.d. background residues, seed 100 + length (reading c13).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

# Robinson & Robinson (1991) background frequencies, NCBI order ARNDCQEGHILKMFPSTWYV.
BG_FREQ = np.array([0.07805, 0.05129, 0.04487, 0.05364, 0.01925, 0.04264, 0.06295, 0.07377,
                    0.02199, 0.05142, 0.09019, 0.05744, 0.02243, 0.03856, 0.05203, 0.07120,
                    0.05841, 0.01330, 0.03216, 0.06441])
BG_CDF = np.cumsum(BG_FREQ / BG_FREQ.sum())
BG_CDF[-1] = 1.0

# The CUDASW++ benchmark query lengths (reading c13), 144 .. 5478.
BENCH_QUERY_LENGTHS = [144, 189, 222, 375, 464, 567, 657, 729, 850, 1000, 1500, 2005,
                       2504, 3005, 3564, 4061, 4548, 4743, 5147, 5478]
C2_QUERY_LENGTHS = [144, 375, 729, 1500, 5478]

MAX_LEN = 35213

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_STREAMS = {"len": 1, "tail": 2, "tailv": 3, "res": 4, "plant": 5, "pmut": 6, "query": 7,
            "rej": 8, "mix": 9, "pwin": 10}


def _splitmix(x: np.ndarray) -> np.ndarray:
    x = x.astype(np.uint64, copy=True)
    with np.errstate(over="ignore"):
        x += np.uint64(0x9E3779B97F4A7C15)
        x = (x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        x = (x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        x = x ^ (x >> np.uint64(31))
    return x


def _key(seed: int, stream: str) -> np.uint64:
    k = _splitmix(np.array([(seed * 0x1000193 + _STREAMS[stream] * 0x9E3779B1) & 0xFFFFFFFFFFFFFFFF],
                           dtype=np.uint64))
    return k[0]


def u01(seed: int, stream: str, idx) -> np.ndarray:
    """Uniform [0,1) doubles, a pure function of (seed, stream, idx)."""
    idx = np.atleast_1d(np.asarray(idx, dtype=np.uint64))
    with np.errstate(over="ignore"):
        x = _splitmix(idx * np.uint64(0xD1B54A32D192ED03) + _key(seed, stream))
    return (x >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def normal(seed: int, stream: str, idx) -> np.ndarray:
    idx = np.asarray(idx, dtype=np.uint64)
    u1 = u01(seed, stream, idx * np.uint64(2))
    u2 = u01(seed, stream, idx * np.uint64(2) + np.uint64(1))
    return np.sqrt(-2.0 * np.log1p(-u1)) * np.cos(2.0 * np.pi * u2)


def background(seed: int, stream: str, idx) -> np.ndarray:
    """i.i.d. background residue codes (0..19) for counter indices idx."""
    return np.searchsorted(BG_CDF, u01(seed, stream, idx), side="right").astype(np.uint8)


# ----------------------------------------------------------------------------- lengths
def sp_lengths(n_seqs: int, seed: int, mu: float = 5.5219, sigma: float = 0.8262,
               tail_frac: float = 1e-4, max_len: int = MAX_LEN) -> np.ndarray:
    """Swiss-Prot-shaped lengths for ALL n_seqs sequences (cheap; every rank computes it)."""
    idx = np.arange(n_seqs, dtype=np.uint64)
    z = normal(seed, "len", idx)
    n = np.clip(np.rint(np.exp(mu + sigma * z)), 2, max_len).astype(np.int64)
    tail = u01(seed, "tail", idx) < tail_frac
    if tail.any():
        lo, hi = np.log(10000.0), np.log(float(max_len))
        tv = np.exp(lo + (hi - lo) * u01(seed, "tailv", idx[tail]))
        n[tail] = np.clip(np.rint(tv), 10000, max_len).astype(np.int64)
    if n_seqs > 0:
        n[int(np.argmax(n))] = max_len
    return n


VARIANCE_STDS = [100, 250, 500, 1000, 2000, 4000]


def variance_lengths(n_seqs: int, std: float, seed: int, max_len: int = 60000) -> np.ndarray:
    """Length-variance workload (Fig.2, L16 §II-C): log-normal lengths with standard
    deviation `std` and mean 1000 + std ("the mean varies" with the deviation), clipped to
    [2, max_len]."""
    mean = 1000.0 + std
    s2 = np.log1p((std / mean) ** 2)
    mu = np.log(mean) - s2 / 2
    z = normal(seed, "len", np.arange(n_seqs, dtype=np.uint64))
    return np.clip(np.rint(np.exp(mu + np.sqrt(s2) * z)), 2, max_len).astype(np.int64)


# PAPER.md L28-L30 Table II: fraction of sequences above T = 3072 (reading c19: ".53%" = 0.53 %)
TABLE2 = [("Ensembl Dog", 0.0053), ("Ensembl Rat", 0.0035), ("RefSeq Human", 0.0056),
          ("RefSeq Mouse", 0.0054), ("TAIR", 0.0006), ("Swiss-Prot", 0.0012)]


def table2_lengths(n_seqs: int, frac_over_3072: float, seed: int) -> np.ndarray:
    """Log-normal lengths with Swiss-Prot's median (mu = 5.5219) and the sigma that puts
    `frac_over_3072` of the sequences at n >= 3072 (one Table II database shape)."""
    from scipy.stats import norm
    sigma = (np.log(3072.0) - 5.5219) / norm.ppf(1.0 - frac_over_3072)
    return sp_lengths(n_seqs, seed, mu=5.5219, sigma=float(sigma), tail_frac=0.0)


def long_lengths(n_seqs: int, seed: int, lo: int = 3073, max_len: int = MAX_LEN,
                 mu: float = 5.5219, sigma: float = 0.8262) -> np.ndarray:
    """Config 3: 90% SP log-normal truncated to [lo, max] by rejection, 10% log-uniform
    [8192, max], one sequence of exactly max_len."""
    idx = np.arange(n_seqs, dtype=np.uint64)
    n = np.zeros(n_seqs, dtype=np.int64)
    pending = np.ones(n_seqs, dtype=bool)
    attempt = 0
    while pending.any():
        pidx = idx[pending]
        z = normal(seed, "rej", pidx * np.uint64(4096) + np.uint64(attempt))
        v = np.rint(np.exp(mu + sigma * z)).astype(np.int64)
        ok = (v >= lo) & (v <= max_len)
        sel = np.nonzero(pending)[0][ok]
        n[sel] = v[ok]
        pending[sel] = False
        attempt += 1
        if attempt > 4000:
            n[pending] = lo
            break
    mix = u01(seed, "mix", idx) < 0.10
    if mix.any():
        a, b = np.log(8192.0), np.log(float(max_len))
        n[mix] = np.clip(np.rint(np.exp(a + (b - a) * u01(seed, "tailv", idx[mix]))), 8192, max_len)
    if n_seqs > 0:
        n[int(np.argmax(n))] = max_len
    return n


# ----------------------------------------------------------------------------- queries
def make_query(length: int, seed: int | None = None) -> np.ndarray:
    s = (100 + length) if seed is None else seed
    return background(s, "query", np.arange(length, dtype=np.uint64))


# ----------------------------------------------------------------------------- database
@dataclass
class Database:
    residues: np.ndarray          # uint8, concatenated codes of THIS shard
    offsets: np.ndarray           # int64 [n+1], CSR into residues
    global_index: np.ndarray      # int64 [n], index of each shard sequence in the full DB
    lengths_all: np.ndarray = field(repr=False, default=None)  # int64 [N], every sequence

    @property
    def num_seqs(self) -> int:
        return int(self.offsets.shape[0] - 1)

    @property
    def lengths(self) -> np.ndarray:
        return np.diff(self.offsets)

    @property
    def total_residues(self) -> int:
        return int(self.offsets[-1])


def shard_indices(lengths_all: np.ndarray, rank: int, world: int) -> np.ndarray:
    """Round-robin over the stable length-descending order; returns the
    global indices of rank's shard in increasing global order."""
    if world == 1:
        return np.arange(lengths_all.shape[0], dtype=np.int64)
    order = np.argsort(-lengths_all, kind="stable")
    return np.sort(order[rank::world]).astype(np.int64)


def build_database(lengths_all: np.ndarray, seed: int, queries=None, plant_frac: float = 1e-4,
                   min_planted: int = 4, sel: np.ndarray | None = None,
                   alphabet_extra: bool = False) -> Database:
    """Generate residues for the sequences `sel` (global indices; default all).

    Residue k of global sequence g is a function of (seed, goff[g] + k) where goff is the
    global CSR offset, so shards are bit-identical to the corresponding slices of the full DB.
    """
    lengths_all = np.asarray(lengths_all, dtype=np.int64)
    n_all = lengths_all.shape[0]
    goff = np.zeros(n_all + 1, dtype=np.int64)
    np.cumsum(lengths_all, out=goff[1:])
    if sel is None:
        sel = np.arange(n_all, dtype=np.int64)
    sel = np.asarray(sel, dtype=np.int64)
    lens = lengths_all[sel]
    off = np.zeros(sel.shape[0] + 1, dtype=np.int64)
    np.cumsum(lens, out=off[1:])
    total = int(off[-1])
    res = np.empty(total, dtype=np.uint8)
    # global residue positions of the shard, generated in bounded chunks
    chunk_seqs = max(1, int(sel.shape[0] // max(1, total // (1 << 24) + 1)))
    for s0 in range(0, sel.shape[0], chunk_seqs):
        s1 = min(sel.shape[0], s0 + chunk_seqs)
        l = lens[s0:s1]
        t = int(l.sum())
        if t == 0:
            continue
        starts = goff[sel[s0:s1]]
        rep = np.repeat(starts - off[s0:s1] + 0, l)  # per-residue global base minus local base
        local = np.arange(off[s0], off[s0] + t, dtype=np.int64)
        gpos = (rep + local).astype(np.uint64)
        res[off[s0]:off[s0] + t] = background(seed, "res", gpos)
    if alphabet_extra:
        # parity-only: sprinkle B, Z, X, * (codes 20..23) at ~2%
        u = u01(seed, "mix", np.arange(total, dtype=np.uint64))
        hit = u < 0.02
        res[hit] = (20 + (u[hit] * 200).astype(np.int64) % 4).astype(np.uint8)
    # planted hits (homologues of the queries), decided per global index
    if queries:
        gidx = np.arange(n_all, dtype=np.uint64)
        up = u01(seed, "plant", gidx)
        planted = np.nonzero(up < plant_frac)[0]
        if planted.shape[0] < min(min_planted, n_all):
            planted = np.argsort(up, kind="stable")[:min(min_planted, n_all)]
        pos_in_shard = {int(g): i for i, g in enumerate(sel)} if sel.shape[0] != n_all else None
        for g in planted:
            g = int(g)
            i = g if pos_in_shard is None else pos_in_shard.get(g)
            if i is None:
                continue
            n = int(lengths_all[g])
            q = np.asarray(queries[g % len(queries)], dtype=np.uint8)
            seq = _planted(q, n, seed, g)
            res[off[i]:off[i] + n] = seq
    return Database(residues=res, offsets=off, global_index=sel, lengths_all=lengths_all)


def _planted(q: np.ndarray, n: int, seed: int, g: int) -> np.ndarray:
    """Window of q with 30% substitutions and 2% indels, embedded in background of length n."""
    base = np.uint64(g) * np.uint64(1 << 20)
    m = q.shape[0]
    wl = min(n, m)
    if wl <= 0:
        return np.zeros(0, dtype=np.uint8)
    start = int(u01(seed, "pwin", np.array([g], dtype=np.uint64))[0] * (m - wl + 1))
    win = q[start:start + wl]
    u = u01(seed, "pmut", base + np.arange(3 * wl, dtype=np.uint64))
    out = []
    for k in range(wl):
        r = u[3 * k]
        if r < 0.01:            # deletion
            continue
        if r < 0.02:            # insertion before this residue
            out.append(int(background(seed, "pmut", base + np.uint64(3 * k + 1))[0]))
        if u[3 * k + 2] < 0.30:  # substitution
            out.append(int(background(seed, "pmut", base + np.uint64(3 * k + 2) + np.uint64(1 << 19))[0]))
        else:
            out.append(int(win[k]))
    out = np.array(out[:n], dtype=np.uint8)
    seq = background(seed, "pmut", base + np.uint64(1 << 18) + np.arange(n, dtype=np.uint64))
    pad = n - out.shape[0]
    lead = pad // 2
    seq[lead:lead + out.shape[0]] = out
    return seq


# ----------------------------------------------------------------------------- configs
@dataclass
class Workload:
    name: str
    db: Database
    queries: list
    matrix_name: str
    gap_open: int
    gap_extend: int
    threshold: int = 3072


def config(name: str, rank: int = 0, world: int = 1, n_override: int | None = None) -> Workload:
    """BASELINE.json configs C1..C5 (SURVEY.md §8(d) "Configs")."""
    if name == "C1":
        qs = [make_query(144)]
        lens = sp_lengths(n_override or 20_000, seed=1)
        db = build_database(lens, 1, qs, sel=shard_indices(lens, rank, world))
        return Workload("C1", db, qs, "BLOSUM62", 10, 2)
    if name in ("C2", "C4"):
        qs = [make_query(L) for L in C2_QUERY_LENGTHS]
        lens = sp_lengths(n_override or 540_000, seed=2)
        db = build_database(lens, 2, qs, sel=shard_indices(lens, rank, world))
        return Workload(name, db, qs, "BLOSUM62", 10, 2)
    if name == "C3":
        qs = [make_query(L) for L in C2_QUERY_LENGTHS]
        lens = long_lengths(n_override or 4096, seed=3)
        db = build_database(lens, 3, qs, sel=shard_indices(lens, rank, world))
        return Workload("C3", db, qs, "BLOSUM62", 10, 2)
    if name == "C5":
        qs = [make_query(L) for L in BENCH_QUERY_LENGTHS]
        lens = sp_lengths(n_override or 50_000_000, seed=5, mu=5.4270)
        db = build_database(lens, 5, qs, sel=shard_indices(lens, rank, world))
        return Workload("C5", db, qs, "BLOSUM45", 10, 2)
    raise ValueError(name)
