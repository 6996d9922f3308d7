"""B200-native Smith-Waterman protein database search (Hains et al., "Improving CUDASW++",
IPDPS 2011) — thin Python binding over the C ABI in include/sw.h.

Argument marshalling only: every step of the search (profile build, both kernels, the
32-bit recompute, the scatter to caller order) runs in libsw_b200.so on the GPU.  There is
no CPU fallback: if the library is missing or the device is not sm_100a, calls raise.

The function names mirror the C ABI: sw_create, sw_set_query, sw_load_db, sw_search,
sw_search_async, sw_search_batch, sw_search_batch_async, sw_last_stats, sw_destroy.
``SmithWaterman`` is a small object wrapper over the same calls.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libsw_b200.so")

SW_OK, SW_E_INVALID, SW_E_STATE, SW_E_NOMEM, SW_E_CUDA, SW_E_UNSUPPORTED = range(6)
SW_AUTO_THRESHOLD = -1
EXPORTED = ["sw_create", "sw_set_query", "sw_load_db", "sw_search", "sw_search_async",
            "sw_search_batch", "sw_search_batch_async", "sw_search_stream", "sw_last_stats", "sw_last_kernel_ms", "sw_last_regime_ms", "sw_last_threshold",
            "sw_align", "sw_top_hits", "sw_destroy",
            "sw_strerror", "sw_last_error", "sw_version"]

_lib = None


class SWError(RuntimeError):
    def __init__(self, status: int, detail: str = ""):
        self.status = status
        super().__init__(f"{_strerror(status)} (status {status}){': ' + detail if detail else ''}")


def load_library(path: str = LIB_PATH):
    """Load libsw_b200.so (raises if it has not been built: there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not built; run `python -m paper_conf_ipps_hainscobr11_b200.build`")
    L = ctypes.CDLL(path)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    L.sw_create.argtypes = [ctypes.POINTER(vp), vp, i32, vp, i32, i32, i32]
    L.sw_set_query.argtypes = [vp, vp, i32]
    L.sw_load_db.argtypes = [vp, vp, i64, vp, i64]
    L.sw_search.argtypes = [vp, vp, i32]
    L.sw_search_async.argtypes = [vp, vp, i32, vp]
    L.sw_search_batch.argtypes = [vp, vp, vp, i32, vp, i32]
    L.sw_search_batch_async.argtypes = [vp, vp, vp, i32, vp, i32, vp]
    L.sw_search_stream.argtypes = [vp, vp, vp, i32, vp, i64, vp, i64, vp, i32, i64]
    L.sw_last_stats.argtypes = [vp, vp]
    L.sw_last_kernel_ms.argtypes = [vp, vp]
    L.sw_last_regime_ms.argtypes = [vp, vp]
    L.sw_last_threshold.argtypes = [vp]
    L.sw_align.argtypes = [vp, i64, vp, vp, i32]
    L.sw_align.restype = ctypes.c_int
    L.sw_top_hits.argtypes = [vp, vp, i64, i32, vp, vp]
    L.sw_top_hits.restype = ctypes.c_int
    L.sw_last_threshold.restype = ctypes.c_int32
    L.sw_destroy.argtypes = [vp]
    L.sw_destroy.restype = None
    L.sw_strerror.argtypes = [ctypes.c_int]
    L.sw_strerror.restype = ctypes.c_char_p
    L.sw_last_error.argtypes = [vp]
    L.sw_last_error.restype = ctypes.c_char_p
    L.sw_version.restype = ctypes.c_char_p
    for name in ("sw_create", "sw_set_query", "sw_load_db", "sw_search", "sw_search_async", "sw_search_batch",
                 "sw_search_batch_async", "sw_search_stream", "sw_last_stats", "sw_last_kernel_ms",
                 "sw_last_regime_ms"):
        getattr(L, name).restype = ctypes.c_int
    _lib = L
    return L


def _strerror(status: int) -> str:
    try:
        return load_library().sw_strerror(status).decode()
    except ImportError:
        return f"status {status}"


def _check(h, status: int):
    if status != SW_OK:
        detail = load_library().sw_last_error(h).decode() if h else ""
        raise SWError(status, detail)


def _u8(a):
    return np.ascontiguousarray(a, dtype=np.uint8)


def sw_create(query, matrix, gap_open: int, gap_extend: int):
    L = load_library()
    q = _u8(query)
    W = np.ascontiguousarray(matrix, dtype=np.int8)
    h = ctypes.c_void_p()
    _check(None, L.sw_create(ctypes.byref(h), q.ctypes.data, int(q.size), W.ctypes.data, int(W.shape[0]),
                             int(gap_open), int(gap_extend)))
    return h


def sw_set_query(h, query):
    q = _u8(query)
    _check(h, load_library().sw_set_query(h, q.ctypes.data, int(q.size)))


def sw_load_db(h, residues, offsets):
    r = _u8(residues)
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    rp = r.ctypes.data if r.size else None
    _check(h, load_library().sw_load_db(h, rp, int(off[-1]), off.ctypes.data, int(off.size - 1)))


def sw_search(h, num_seqs: int, length_threshold: int = 3072) -> np.ndarray:
    out = np.zeros(max(num_seqs, 1), dtype=np.int32)
    _check(h, load_library().sw_search(h, out.ctypes.data, int(length_threshold)))
    return out[:num_seqs]


def sw_search_async(h, d_scores_ptr: int, length_threshold: int, stream_ptr: int = 0):
    _check(h, load_library().sw_search_async(h, ctypes.c_void_p(d_scores_ptr), int(length_threshold),
                                             ctypes.c_void_p(stream_ptr)))


def _batch(queries):
    qs = [_u8(q) for q in queries]
    off = np.zeros(len(qs) + 1, dtype=np.int64)
    off[1:] = np.cumsum([q.size for q in qs])
    cat = np.concatenate(qs) if qs else np.zeros(1, np.uint8)
    return np.ascontiguousarray(cat), off


def sw_search_batch(h, queries, num_seqs: int, length_threshold: int = 3072, out=None) -> np.ndarray:
    """out: an optional int32 [len(queries), num_seqs] C-contiguous host array to fill (e.g. pinned
    memory reused across calls: the copies then run at full rate with no page faults)."""
    cat, off = _batch(queries)
    if out is not None:
        if (out.dtype != np.int32 or not out.flags.c_contiguous or out.shape != (len(queries), num_seqs)
                or num_seqs == 0):
            raise ValueError("out must be a C-contiguous int32 array of shape (len(queries), num_seqs)")
    else:
        out = np.zeros((len(queries), max(num_seqs, 1)), dtype=np.int32)
    _check(h, load_library().sw_search_batch(h, cat.ctypes.data, off.ctypes.data, len(queries), out.ctypes.data,
                                              int(length_threshold)))
    return out[:, :num_seqs]


def sw_search_batch_async(h, queries, d_scores_ptr: int, length_threshold: int, stream_ptr: int = 0):
    cat, off = _batch(queries)
    _check(h, load_library().sw_search_batch_async(h, cat.ctypes.data, off.ctypes.data, len(queries),
                                                   ctypes.c_void_p(d_scores_ptr), int(length_threshold),
                                                   ctypes.c_void_p(stream_ptr)))


def sw_search_stream(h, residues, offsets, length_threshold: int = 3072, chunk_residues: int = 1 << 28,
                     queries=None) -> np.ndarray:
    """Search a host-resident database chunk by chunk, uploads overlapped with the search.
    queries=None: the handle's query, returns int32[num_seqs]; else int32[len(queries), num_seqs]."""
    r = _u8(residues)
    off = np.ascontiguousarray(offsets, dtype=np.int64)
    n = int(off.size - 1)
    rp = r.ctypes.data if r.size else None
    if queries is None:
        qp, op, nq = None, None, 1
    else:
        cat, qoff = _batch(queries)
        qp, op, nq = cat.ctypes.data, qoff.ctypes.data, len(queries)
    out = np.zeros((nq, max(n, 1)), dtype=np.int32)
    _check(h, load_library().sw_search_stream(h, qp, op, nq, rp, int(off[-1]), off.ctypes.data, n, out.ctypes.data,
                                              int(length_threshold), int(chunk_residues)))
    return out[0, :n] if queries is None else out[:, :n]


def sw_last_stats(h) -> dict:
    out = np.zeros(4, dtype=np.int64)
    _check(h, load_library().sw_last_stats(h, out.ctypes.data))
    return {"recomputed_s32": int(out[0]), "long_seqs": int(out[1]), "short_seqs": int(out[2]),
            "launches": int(out[3])}


def sw_last_kernel_ms(h) -> dict:
    out = np.zeros(2, dtype=np.float64)
    _check(h, load_library().sw_last_kernel_ms(h, out.ctypes.data))
    return {"search_ms": float(out[0]), "recompute_ms": float(out[1])}


def sw_last_regime_ms(h) -> dict:
    out = np.zeros(3, dtype=np.float64)
    _check(h, load_library().sw_last_regime_ms(h, out.ctypes.data))
    return {"long_ms": float(out[0]), "search_ms": float(out[1]), "fused_long_queries": int(out[2])}


class Alignment(ctypes.Structure):
    _fields_ = [("score", ctypes.c_int32), ("q_begin", ctypes.c_int32), ("q_end", ctypes.c_int32),
                ("d_begin", ctypes.c_int32), ("d_end", ctypes.c_int32), ("n_ops", ctypes.c_int32)]


OPS = "MID"


def sw_align(h, seq_index: int, ops_cap: int = 1 << 16) -> dict:
    """Optimal local alignment (device traceback) of the handle's query with one sequence."""
    L = load_library()
    out = Alignment()
    ops = np.zeros(max(ops_cap, 1), dtype=np.uint32)
    st = L.sw_align(h, int(seq_index), ctypes.byref(out), ops.ctypes.data, int(ops_cap))
    if st != SW_OK and out.n_ops > ops_cap:
        return sw_align(h, seq_index, int(out.n_ops))
    _check(h, st)
    runs = [(OPS[int(v) & 3], int(v) >> 2) for v in ops[: out.n_ops]]
    return {"score": out.score, "q_begin": out.q_begin, "q_end": out.q_end, "d_begin": out.d_begin,
            "d_end": out.d_end, "runs": runs, "cigar": "".join(f"{n}{o}" for o, n in runs)}


def sw_top_hits(h, scores, k: int):
    """The k best (index, score) of a score array, best first (ties: smaller index), selected
    on the device."""
    sc = np.ascontiguousarray(scores, dtype=np.int32).reshape(-1)
    kk = max(0, min(int(k), sc.size))
    idx = np.zeros(max(kk, 1), dtype=np.int64)
    val = np.zeros(max(kk, 1), dtype=np.int32)
    _check(h, load_library().sw_top_hits(h, sc.ctypes.data, sc.size, int(k), idx.ctypes.data, val.ctypes.data))
    return idx[:kk], val[:kk]


def sw_destroy(h):
    if h:
        load_library().sw_destroy(h)


class SmithWaterman:
    """Object wrapper: one query + scoring scheme, one loaded database (caller order kept)."""

    def __init__(self, query, matrix, gap_open: int, gap_extend: int):
        self.h = sw_create(query, matrix, gap_open, gap_extend)
        self.num_seqs = 0

    def set_query(self, query):
        sw_set_query(self.h, query)

    def load_db(self, residues, offsets):
        sw_load_db(self.h, residues, offsets)
        self.num_seqs = int(np.asarray(offsets).shape[0] - 1)

    def search(self, length_threshold: int = 3072) -> np.ndarray:
        return sw_search(self.h, self.num_seqs, length_threshold)

    def search_batch(self, queries, length_threshold: int = 3072, out=None) -> np.ndarray:
        return sw_search_batch(self.h, queries, self.num_seqs, length_threshold, out)

    def search_batch_into(self, queries, d_scores_ptr: int, length_threshold: int = 3072, stream_ptr: int = 0):
        sw_search_batch_async(self.h, queries, d_scores_ptr, length_threshold, stream_ptr)

    def search_stream(self, residues, offsets, length_threshold: int = 3072, chunk_residues: int = 1 << 28,
                      queries=None):
        return sw_search_stream(self.h, residues, offsets, length_threshold, chunk_residues, queries)

    def stats(self) -> dict:
        return sw_last_stats(self.h)

    def kernel_ms(self) -> dict:
        return sw_last_kernel_ms(self.h)

    def regime_ms(self) -> dict:
        return sw_last_regime_ms(self.h)

    def align(self, seq_index: int) -> dict:
        return sw_align(self.h, seq_index)

    def top_hits(self, scores, k: int):
        return sw_top_hits(self.h, scores, k)

    def last_threshold(self) -> int:
        return int(load_library().sw_last_threshold(self.h))

    def close(self):
        if self.h:
            sw_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
