"""C-ABI contract tests that need no GPU (T2): the library loads, exports
every symbol include/krcv.h declares, and the host-only entry points and
host-side validation behave as documented.  No compute call is made."""
from __future__ import annotations

import ctypes
import math
import os
import re

import numpy as np
import pytest

import workloads
from paper_conf_ipps_rohlfsz17_b200 import krcv

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "krcv.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(kr_[a-z_]+)\s*\(", src)))


def test_header_declares_exports_and_library_has_them():
    declared = _declared()
    assert set(declared) == set(krcv.EXPORTS), declared
    lib = ctypes.CDLL(krcv.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name


def test_library_is_sm100a_only():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {krcv.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out
    assert "sm_90" not in out and "sm_80" not in out


def test_version_and_strerror():
    assert "sm_100a" in krcv.kr_version()
    for st in range(8):
        assert isinstance(krcv.kr_strerror(st), str) and krcv.kr_strerror(st)
    assert krcv.kr_strerror(99) == "unknown status"


@pytest.mark.parametrize("m", [1, 7, 100, 1000])
def test_default_grid_matches_recipe(m):
    x, _ = workloads.draw_xy("paper", 513, 4)
    h = krcv.kr_default_grid(x, m)
    assert np.array_equal(h, workloads.grid_default(x, m))
    assert h[-1] == x.max() - x.min()


def test_default_grid_errors():
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_default_grid(np.ones(8), 3)
    assert e.value.status == krcv.KR_EDEGENERATE
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_default_grid(np.array([0.0, math.nan]), 3)
    assert e.value.status == krcv.KR_ENONFINITE
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_default_grid(np.array([0.0]), 3)
    assert e.value.status == krcv.KR_EARG


@pytest.mark.parametrize("h,code", [
    ([0.1, 0.2], krcv.KR_OK), ([0.2, 0.2], krcv.KR_OK), ([0.2, 0.1], krcv.KR_EGRID),
    ([0.0], krcv.KR_EGRID), ([-1.0], krcv.KR_EGRID), ([math.nan], krcv.KR_EGRID),
    ([math.inf], krcv.KR_EGRID), ([], krcv.KR_EARG)])
def test_validate_grid(h, code):
    assert krcv.kr_validate_grid(np.array(h, np.float64)) == code


def test_validate_grid_max_m():
    assert krcv.kr_validate_grid(np.linspace(0.1, 1, krcv.KR_MAX_M)) == krcv.KR_OK
    assert krcv.kr_validate_grid(np.linspace(0.1, 1, krcv.KR_MAX_M + 1)) == krcv.KR_EARG


@pytest.mark.parametrize("bad,code", [
    (dict(x=[0.0], y=[1.0]), krcv.KR_EARG),
    (dict(kernel=9), krcv.KR_EKERNEL),
    (dict(h=[0.5, 0.25]), krcv.KR_EGRID),
])
def test_cv_grid_host_validation_before_device(bad, code):
    """Arguments and the grid are validated before any CUDA call (works
    without a GPU); outputs are untouched on error.  (NaN / Inf in x, y are
    detected on the device: tests/test_gpu_parity.py
    test_host_api_nonfinite_and_graph_replay.)"""
    a = dict(x=[0.0, 0.5, 1.0], y=[1.0, 2.0, 3.0], h=[0.5, 1.0], kernel=1)
    a.update(bad)
    x, y, h = (np.array(a[k], np.float64) for k in ("x", "y", "h"))
    cv = np.full(h.shape[0], 7.0)
    best = ctypes.c_int32(-5)
    st = krcv._lib().kr_cv_grid(x.ctypes.data, y.ctypes.data, x.shape[0], h.ctypes.data, h.shape[0],
                                a["kernel"], cv.ctypes.data, ctypes.byref(best))
    assert st == code
    assert np.all(cv == 7.0) and best.value == -5


def test_null_pointers():
    lib = krcv._lib()
    assert lib.kr_cv_grid(None, None, 10, None, 3, 1, None, None) == krcv.KR_EARG
    assert lib.kr_cv_shard_async(None, None, 10, None, 3, 1, 0, 1, None, None, 0, None) == krcv.KR_EARG
    assert lib.kr_finalize(None, 10, 3, None, None, None) == krcv.KR_EARG
    assert lib.kr_finalize_async(None, 10, 3, None, None, None, None, None) == krcv.KR_EARG


def test_shard_argument_checks_without_device():
    """Argument errors of the async entry point are host-side (no GPU needed)."""
    lib = krcv._lib()
    p = ctypes.c_void_p(256)  # never dereferenced: rejected before any launch
    assert lib.kr_cv_shard_async(p, p, 1, p, 3, 1, 0, 1, p, p, 1 << 20, None) == krcv.KR_EARG
    assert lib.kr_cv_shard_async(p, p, 10, p, 3, 5, 0, 1, p, p, 1 << 20, None) == krcv.KR_EKERNEL
    assert lib.kr_cv_shard_async(p, p, 10, p, 3, 1, 2, 2, p, p, 1 << 20, None) == krcv.KR_EARG
    assert lib.kr_cv_shard_async(p, p, 10, p, 3, 1, 0, 0, p, p, 1 << 20, None) == krcv.KR_EARG
    assert lib.kr_cv_shard_async(p, p, 10, p, 0, 1, 0, 1, p, p, 1 << 20, None) == krcv.KR_EARG
    assert lib.kr_cv_shard_async(p, p, 10, ctypes.c_void_p(257), 3, 1, 0, 1, p, ctypes.c_void_p(257),
                                 1 << 20, None) == krcv.KR_EARG  # misaligned workspace


def test_host_finalize_rules():
    m = 4
    S = np.array([3.0, 1.0, 1.0, 2.0])
    neff = np.array([5.0, 5.0, 6.0, 6.0])
    part = np.concatenate([S, neff, [0.0, 0.0]])
    cv, ne, best = krcv.kr_finalize(part, 2, m)
    assert np.array_equal(cv, S / 2) and list(ne) == [5, 5, 6, 6] and best == 1  # ties -> lowest
    part[0] = math.nan
    assert krcv.kr_finalize(part, 2, m)[2] == 1  # NaN never minimal
    part[2 * m] = 1.0
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_finalize(part, 2, m)
    assert e.value.status == krcv.KR_EGRID
    part[2 * m] = 0.0
    part[2 * m + 1] = 3.0
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_finalize(part, 2, m)
    assert e.value.status == krcv.KR_ENONFINITE


def test_product_does_not_import_oracle():
    """The product path never touches oracle/ (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_rohlfsz17_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src
                assert "kr_oracle" not in src and "kro_" not in src
