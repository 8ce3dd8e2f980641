"""The synchronous host-pointer path (kr_cv_grid*, krcv_host.cpp) keeps device
buffers, a pinned result staging block and -- for pinned caller buffers -- a
captured CUDA graph between calls.  A call that grows any of those buffers
must drop the graph: the graph's nodes point at the old
allocations.  Each case below interleaves calls that reallocate with repeat
pinned calls and checks every result against the oracle (Program 3,
oracle.cv_sorted), curve and n_eff element by element."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import workloads
from tests.helpers import best_ok, cv_rel_err

pytestmark = pytest.mark.gpu

TOL = 1e-10


def _pinned(a):
    import torch

    t = torch.from_numpy(np.ascontiguousarray(a, np.float64)).pin_memory()
    return t, t.numpy()  # the numpy view shares the pinned allocation


def _check(x, y, h, k, got):
    cv, neff, best = got
    ref = oracle.cv_sorted(x, y, h, k)
    assert cv_rel_err(cv, ref.cv) <= TOL
    assert np.array_equal(neff, ref.neff)
    assert best_ok(best, ref.cv)


@pytest.mark.parametrize("order", ["pageable_grows_n", "pageable_grows_m", "refine_grows", "kde_grows"])
def test_pinned_replay_after_reallocation(order):
    from paper_conf_ipps_rohlfsz17_b200 import krcv

    krcv.kr_release()  # start from an empty host context
    x1, y1, h1, k = workloads.make("C2", seed=3, n=1000)
    h1 = h1[:50]
    keep = [_pinned(a) for a in (x1, y1, h1)]
    px, py, ph = (v[1] for v in keep)
    _check(x1, y1, h1, k, krcv.kr_cv_grid(px, py, ph, k, with_neff=True))  # captures the graph
    _check(x1, y1, h1, k, krcv.kr_cv_grid(px, py, ph, k, with_neff=True))  # replays it
    if order == "pageable_grows_n":
        x2, y2, h2, _ = workloads.make("C2", seed=4, n=5000)
        _check(x2, y2, h2[:50], k, krcv.kr_cv_grid(x2, y2, h2[:50], k, with_neff=True))
    elif order == "pageable_grows_m":
        x2, y2, h2, _ = workloads.make("C2", seed=4, n=1000)
        _check(x2, y2, h2, k, krcv.kr_cv_grid(x2, y2, h2, k, with_neff=True))  # m = 200 > 50
    elif order == "refine_grows":
        x2, y2, h2, _ = workloads.make("C2", seed=4, n=4000)
        krcv.kr_cv_refine(x2, y2, h2, k, levels=2, m_fine=129)
    else:
        x2, _, h2, _ = workloads.make("C2", seed=4, n=6000)
        krcv.kr_kde_lscv(x2, h2, "epanechnikov")
    # the repeat pinned call: same caller pointers, n, m, kernel -- must not
    # replay a graph that points at freed buffers
    for _ in range(2):
        _check(x1, y1, h1, k, krcv.kr_cv_grid(px, py, ph, k, with_neff=True))
    # and new values in the same pinned buffers are read at replay time
    x3, y3, _, _ = workloads.make("C2", seed=5, n=1000)
    px[:] = x3
    py[:] = y3
    _check(x3, y3, h1, k, krcv.kr_cv_grid(px, py, ph, k, with_neff=True))
    del keep
