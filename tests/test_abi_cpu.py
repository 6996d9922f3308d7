"""CPU-side checks of the boundary: the C-ABI library builds, loads and exports every
symbol include/sw.h declares; calls that need no GPU behave as documented."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_hainscobr11_b200 as swp
from paper_conf_ipps_hainscobr11_b200 import build as swbuild

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    txt = open(os.path.join(ROOT, "include", "sw.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(sw_[a-z_]+)\s*\(", txt)))


def test_library_builds_and_exports_every_declared_symbol():
    path = swbuild.build()
    L = ctypes.CDLL(path)
    names = _declared()
    assert set(names) == set(swp.EXPORTED)
    for n in names:
        assert hasattr(L, n), n


def test_strerror_and_version():
    L = swp.load_library()
    for s, txt in [(0, "ok"), (1, "invalid argument"), (2, "call out of order"), (3, "out of memory"),
                   (4, "CUDA error"), (5, "unsupported device or parameters")]:
        assert L.sw_strerror(s).decode() == txt
    assert b"sm_100a" in L.sw_version()
    assert L.sw_last_error(None) == b""


def test_null_safety_without_gpu():
    L = swp.load_library()
    L.sw_destroy(None)                       # NULL-safe
    assert L.sw_search(None, None, 0) == swp.SW_E_INVALID
    assert L.sw_load_db(None, None, 0, None, 0) == swp.SW_E_INVALID
    assert L.sw_create(None, None, 0, None, 0, 0, 0) == swp.SW_E_INVALID


def test_create_validates_before_touching_the_device():
    q = np.array([0, 1, 2], np.uint8)
    W = np.eye(4, dtype=np.int8)
    with pytest.raises(swp.SWError) as e:
        swp.sw_create(q, W, -1, 2)                     # negative gap open
    assert e.value.status == swp.SW_E_INVALID
    with pytest.raises(swp.SWError) as e:
        swp.sw_create(np.array([7], np.uint8), W, 1, 1)  # code >= alphabet
    assert e.value.status == swp.SW_E_INVALID
    with pytest.raises(swp.SWError) as e:
        swp.sw_create(q, W, 127, 1)                    # rho + max_w > 127: outside the s16 profile range
    assert e.value.status == swp.SW_E_UNSUPPORTED


def test_no_cpu_fallback_without_device():
    """With no sm_100 device the library refuses (SW_E_UNSUPPORTED) instead of computing."""
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    with pytest.raises(swp.SWError) as e:
        swp.sw_create(np.array([0, 1], np.uint8), np.eye(4, dtype=np.int8), 10, 2)
    assert e.value.status == swp.SW_E_UNSUPPORTED
