"""C-ABI contract on the GPU (include/sw.h): one test per error code / state rule, ownership
(inputs copied), the device-pointer stream-ordered entry points and the statistics calls."""
import ctypes

import numpy as np
import pytest

import oracle
import paper_conf_ipps_hainscobr11_b200 as swp
from workloads import gen
from workloads.matrices import BLOSUM62

pytestmark = pytest.mark.gpu


def _db(n=200, seed=4):
    return gen.build_database(gen.sp_lengths(n, seed=seed), seed)


def test_search_before_load_is_state_error():
    h = swp.sw_create(gen.make_query(50), BLOSUM62, 10, 2)
    try:
        with pytest.raises(swp.SWError) as e:
            swp.sw_search(h, 1, 3072)
        assert e.value.status == swp.SW_E_STATE
    finally:
        swp.sw_destroy(h)


def test_invalid_arguments():
    L = swp.load_library()
    h = swp.sw_create(gen.make_query(50), BLOSUM62, 10, 2)
    try:
        res = np.zeros(10, np.uint8)
        bad_off = np.array([0, 5, 3, 10], np.int64)          # not non-decreasing
        assert L.sw_load_db(h, res.ctypes.data, 10, bad_off.ctypes.data, 3) == swp.SW_E_INVALID
        bad_off2 = np.array([1, 5, 10], np.int64)            # offsets[0] != 0
        assert L.sw_load_db(h, res.ctypes.data, 10, bad_off2.ctypes.data, 2) == swp.SW_E_INVALID
        bad_res = np.full(10, 30, np.uint8)                   # code >= alphabet
        off = np.array([0, 10], np.int64)
        assert L.sw_load_db(h, bad_res.ctypes.data, 10, off.ctypes.data, 1) == swp.SW_E_INVALID
        assert b"alphabet" in L.sw_last_error(h)
        swp.sw_load_db(h, np.zeros(10, np.uint8), off)
        out = np.zeros(1, np.int32)
        assert L.sw_search(h, out.ctypes.data, -2) == swp.SW_E_INVALID   # T < 0 (and not SW_AUTO_THRESHOLD)
        assert L.sw_search(h, None, 10) == swp.SW_E_INVALID             # NULL output
        q = np.array([1, 2, 99], np.uint8)
        assert L.sw_set_query(h, q.ctypes.data, 3) == swp.SW_E_INVALID   # bad query code
        assert L.sw_set_query(h, q.ctypes.data, 0) == swp.SW_E_INVALID   # empty query
    finally:
        swp.sw_destroy(h)


def test_inputs_are_copied_and_reload_replaces_db():
    db = _db()
    q = gen.make_query(120)
    h = swp.sw_create(q, BLOSUM62, 10, 2)
    try:
        res = db.residues.copy()
        swp.sw_load_db(h, res, db.offsets)
        res[:] = 0                      # caller reuses its buffer: the library owns a copy
        q[:] = 0
        out = swp.sw_search(h, db.num_seqs, 3072)
        ref = oracle.scores(gen.make_query(120), BLOSUM62, 10, 2, db.residues, db.offsets)
        assert np.array_equal(out, ref)
        db2 = _db(50, seed=9)
        swp.sw_load_db(h, db2.residues, db2.offsets)
        out2 = swp.sw_search(h, db2.num_seqs, 3072)
        assert out2.shape == (50,)
        assert np.array_equal(out2, oracle.scores(gen.make_query(120), BLOSUM62, 10, 2, db2.residues, db2.offsets))
    finally:
        swp.sw_destroy(h)


def test_async_device_pointer_and_stream():
    import torch
    db = _db()
    q = gen.make_query(333)
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        st = torch.cuda.Stream()
        out = torch.full((db.num_seqs,), -7, dtype=torch.int32, device="cuda")
        swp.sw_search_async(sw.h, out.data_ptr(), 3072, st.cuda_stream)
        st.synchronize()
        ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets)
        assert np.array_equal(out.cpu().numpy(), ref)
        # batch into a device tensor, joined back into the caller's stream
        qs = [gen.make_query(L) for L in (144, 375, 5)]
        outb = torch.full((3, db.num_seqs), -1, dtype=torch.int32, device="cuda")
        sw.search_batch_into(qs, outb.data_ptr(), 3072, st.cuda_stream)
        st.synchronize()
        for k, qq in enumerate(qs):
            assert np.array_equal(outb[k].cpu().numpy(), oracle.scores(qq, BLOSUM62, 10, 2, db.residues, db.offsets))
        stats = sw.stats()
        assert stats["launches"] > 0 and stats["recomputed_s32"] == 0
        km = sw.kernel_ms()
        assert km["search_ms"] > 0


def test_formerly_unsupported_parameter_ranges_now_search():
    """Round 1 refused rho + max(w) > 127 (the int8 profile range) and queries whose profile does
    not fit shared memory; both now run (WIDE kernels, long-query mode) with exact scores —
    and never on the CPU (tests/test_wide_params_gpu.py, tests/test_long_query_gpu.py)."""
    import oracle
    db = _db(20)
    for q, rho in ((gen.make_query(10), 120), (gen.make_query(20000), 10)):
        h = swp.sw_create(q, BLOSUM62, rho, 1)
        try:
            swp.sw_load_db(h, db.residues, db.offsets)
            got = swp.sw_search(h, db.num_seqs, 3072)
        finally:
            swp.sw_destroy(h)
        assert np.array_equal(got, oracle.scores(q, BLOSUM62, rho, 1, db.residues, db.offsets))


def test_version_and_null_destroy():
    L = swp.load_library()
    assert L.sw_version().startswith(b"sw_b200")
    L.sw_destroy(ctypes.c_void_p())


@pytest.mark.parametrize("chunk", [1, 997, 20000, 1 << 30])
def test_search_stream_matches_oracle(chunk):
    """sw_search_stream (f3): chunked, upload-overlapped search == oracle for any chunk size,
    including one sequence per chunk and a single chunk; the loaded database is untouched."""
    db = gen.build_database(np.concatenate([gen.sp_lengths(900, seed=12), [4000, 0, 3500, 1]]), 12)
    q = gen.make_query(222)
    ref = oracle.scores(q, BLOSUM62, 10, 2, db.residues, db.offsets)
    other = _db(30, seed=2)
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(other.residues, other.offsets)
        out = sw.search_stream(db.residues, db.offsets, 3072 if chunk != 997 else swp.SW_AUTO_THRESHOLD, chunk)
        assert np.array_equal(out, ref)
        assert sw.stats()["long_seqs"] + sw.stats()["short_seqs"] == db.num_seqs
        assert np.array_equal(sw.search(3072), oracle.scores(q, BLOSUM62, 10, 2, other.residues, other.offsets))
        qs = [gen.make_query(L) for L in (7, 300, 1200)]
        outb = sw.search_stream(db.residues, db.offsets, 3072, chunk, queries=qs)
        for k, qq in enumerate(qs):
            assert np.array_equal(outb[k], oracle.scores(qq, BLOSUM62, 10, 2, db.residues, db.offsets))


def test_search_stream_growing_chunks_match_resident():
    """Chunks of growing size force the device database buffers of a stream slot to be
    reallocated while the other slot's search runs: the streamed scores must equal the
    resident search bit for bit (regression: a zero-fill of freshly allocated buffers on the
    legacy stream raced the upload stream and corrupted chunks)."""
    lens = gen.sp_lengths(60_000, seed=21)
    lens[::7] += np.arange(lens[::7].size) % 700            # later chunks hold longer sequences
    db = gen.build_database(np.sort(lens), 21)
    q = gen.make_query(5478)
    with swp.SmithWaterman(q, BLOSUM62, 10, 2) as sw:
        sw.load_db(db.residues, db.offsets)
        ref = sw.search(3072)
        for chunk in (1 << 20, 3 << 20):
            assert np.array_equal(sw.search_stream(db.residues, db.offsets, 3072, chunk).reshape(-1), ref)


def test_search_stream_errors_and_empty():
    L = swp.load_library()
    with swp.SmithWaterman(gen.make_query(40), BLOSUM62, 10, 2) as sw:
        out = sw.search_stream(np.zeros(0, np.uint8), np.array([0], np.int64))
        assert out.shape == (0,)
        res = np.zeros(10, np.uint8)
        off = np.array([0, 10], np.int64)
        sc = np.zeros(1, np.int32)
        def call(roff=off, out=sc, chunk=64, qs=None, qo=None, nq=1):
            return L.sw_search_stream(sw.h, qs, qo, nq, res.ctypes.data, 10, roff.ctypes.data, 1, out, 3072, chunk)
        assert call(out=sc.ctypes.data, chunk=0) == swp.SW_E_INVALID
        assert call(roff=np.array([0, 11], np.int64), out=sc.ctypes.data) == swp.SW_E_INVALID
        assert call(out=None) == swp.SW_E_INVALID
        badq, qo = np.array([1, 40], np.uint8), np.array([0, 2], np.int64)
        assert call(out=sc.ctypes.data, qs=badq.ctypes.data, qo=qo.ctypes.data) == swp.SW_E_INVALID
        assert call(out=sc.ctypes.data) == swp.SW_OK and sc[0] == oracle.scores(
            gen.make_query(40), BLOSUM62, 10, 2, res, off)[0]
        # overflow counts are summed over chunks
        hp = np.full(3000, 17, np.uint8)              # W-W = 11: 33000 > int16
        sw.set_query(hp)
        out = sw.search_stream(np.concatenate([hp, hp]), np.array([0, 3000, 6000], np.int64), 3072, 3000)
        assert list(out) == [3000 * int(BLOSUM62[17, 17])] * 2 and sw.stats()["recomputed_s32"] == 2
