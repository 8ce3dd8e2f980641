"""Fault injection (SURVEY.md §5 "failure detection"): KRCV_FAIL_AT=<stage>
makes the enqueue stop before that stage and return KR_ECUDA with the stage
named in kr_last_cuda_error.  Checks the error unwinding of every entry
point that runs the stage: the call fails cleanly (no output written through
the raw ABI), and the next call without the hook returns the clean result
bit for bit (no state left behind: status words, completion counter, the
captured host-path graph)."""
from __future__ import annotations

import ctypes
import os

import numpy as np
import pytest

from paper_conf_ipps_rohlfsz17_b200 import krcv

pytestmark = pytest.mark.gpu


def _data(n=3000, seed=5):
    rng = np.random.default_rng(seed)
    x = rng.uniform(0, 1, n)
    y = 0.5 * x + 10 * x * x + rng.uniform(0, 0.5, n)
    return x, y, krcv.kr_default_grid(x, 24)


@pytest.mark.parametrize("algo", ["prefix", "sweep", "hist"])
@pytest.mark.parametrize("stage", ["sort", "prefix", "sweep", "reduce"])
def test_injected_failure_unwinds(monkeypatch, stage, algo):
    x, y, h = _data()
    clean_cv, clean_best = krcv.kr_cv_grid(x, y, h, "epanechnikov", algo=algo)
    monkeypatch.setenv("KRCV_FAIL_AT", stage)
    cv = np.full(h.size, -7.0)
    best = ctypes.c_int32(-5)
    st = krcv._lib().kr_cv_grid_algo(x.ctypes.data, y.ctypes.data, x.size, h.ctypes.data, h.size, 1,
                                      krcv._algo_id(algo), cv.ctypes.data, None, ctypes.byref(best))
    if stage == "prefix" and algo != "prefix":  # no prefix build on this path
        assert st == 0
    else:
        assert st == krcv.KR_ECUDA
        assert stage in krcv._lib().kr_last_cuda_error().decode()
        assert np.all(cv == -7.0) and best.value == -5  # outputs untouched
    monkeypatch.delenv("KRCV_FAIL_AT")
    cv2, best2 = krcv.kr_cv_grid(x, y, h, "epanechnikov", algo=algo)
    if algo != "hist":  # the histogram's fp64 shared-memory atomics are order-dependent
        assert np.array_equal(cv2.view(np.uint64), clean_cv.view(np.uint64))
    else:
        assert np.allclose(cv2, clean_cv, rtol=1e-12, atol=0)
    assert best2 == clean_best


def test_injected_failure_pinned_graph_path(monkeypatch):
    """The pinned-buffer host path captures a CUDA graph: a failure during the
    capture must not leave a half-built graph behind."""
    torch = pytest.importorskip("torch")
    x, y, h = _data(2000, 9)
    hx, hy, hh = (torch.from_numpy(a).pin_memory() for a in (x, y, h))
    hcv = torch.empty(h.size, dtype=torch.float64).pin_memory()
    best = ctypes.c_int32(-1)
    call = lambda: krcv.kr_cv_grid_ptr(hx.data_ptr(), hy.data_ptr(), x.size, hh.data_ptr(), h.size, 1,
                                       hcv.data_ptr(), ctypes.byref(best))
    assert call() == 0
    ref = hcv.numpy().copy()
    krcv.kr_release()  # force a fresh capture on the next call
    monkeypatch.setenv("KRCV_FAIL_AT", "sweep")
    assert call() == krcv.KR_ECUDA
    monkeypatch.delenv("KRCV_FAIL_AT")
    hcv.fill_(0.0)
    assert call() == 0
    assert np.array_equal(hcv.numpy().view(np.uint64), ref.view(np.uint64))
    assert call() == 0  # replay of the re-captured graph
    assert np.array_equal(hcv.numpy().view(np.uint64), ref.view(np.uint64))
