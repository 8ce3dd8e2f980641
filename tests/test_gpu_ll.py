"""GPU parity of the local-linear LOO-CV path (reading Q25; krcv_ll.cuh)
through the C-ABI vs the oracle's plain WLS-intercept definition
(oracle.ll_cv, long double; itself pinned in tests/test_oracle_pins.py).

Bar: the north_star's 1e-6 relative on CV(h) and identical best (tie rule);
on these well-conditioned workloads the tests assert 1e-10.  n_eff (rows with
>= 2 distinct x in the window) is integer work and must match exactly.
"""
from __future__ import annotations

import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import workloads
from paper_conf_ipps_rohlfsz17_b200 import krcv
from paper_conf_ipps_rohlfsz17_b200.api import cv_grid
from tests.helpers import best_ok, cv_rel_err

pytestmark = pytest.mark.gpu

U, E, T, GA = 0, 1, 2, 3
TIGHT = 1e-10


def _check(x, y, h, k, tol=TIGHT):
    cv, neff, best = krcv.kr_ll_cv_grid(x, y, h, k, with_neff=True)
    ref = oracle.ll_cv(x, y, h, k)
    err = cv_rel_err(cv, ref.cv)
    assert err <= tol, err
    assert np.array_equal(neff, ref.neff)
    assert best_ok(best, ref.cv), (best, ref.best)
    return err


def test_ll_worked_example():
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "ll_worked_example.json")))
    for case in g["cases"]:
        k = workloads.KERNEL_IDS[case["kernel"]]
        cv, neff, _ = krcv.kr_ll_cv_grid(g["x"], g["y"], [case["h"]], k, with_neff=True)
        want = float(Fraction(case["cv"]))
        assert abs(cv[0] - want) <= 4 * math.ulp(want) if want else cv[0] == 0.0
        assert int(neff[0]) == case["neff"]


@pytest.mark.parametrize("k", [U, E, T])
@pytest.mark.parametrize("dist,n", [("paper", 2), ("paper", 3), ("paper", 65), ("paper", 1000),
                                    ("sin_uniform", 777), ("lognormal", 900)])
def test_ll_parity(k, dist, n):
    """Small and ragged n (several 32-row tiles plus a tail), both the direct
    (windows <= 16 points) and the prefix (dd moments) branches."""
    x, y = workloads.draw_xy(dist, n, 31)
    m = 37
    h = workloads.grid_log(x, m) if dist == "lognormal" else workloads.grid_default(x, m)
    _check(x, y, h, k)


@pytest.mark.parametrize("k", [U, E, T])
def test_ll_duplicates_and_dyadic(k):
    """Heavy duplicates (M = 0 windows holding one x value, d = 0 neighbours)
    and dyadic inputs with points exactly at h."""
    rng = np.random.default_rng(5)
    x = np.round(rng.uniform(0, 4, 600) * 8) / 8
    y = np.round(rng.normal(0, 1, 600) * 16) / 16
    h = np.array([0.0625, 0.125, 0.1875, 0.25, 0.5, 1.0, 4.0])
    _check(x, y, h, k)
    for seed in range(6):
        xs, ys, hs = workloads.random_dyadic(int(rng.integers(2, 40)), 5, 900 + seed)
        _check(xs, ys, hs, k)


@pytest.mark.parametrize("k", [U, E, T])
def test_ll_reproduces_lines(k):
    """y = a + b x: every counted LOO residual is 0 up to fp64 rounding."""
    x, _ = workloads.draw_xy("paper", 3000, 8)
    y = 0.75 - 2.5 * x
    h = workloads.grid_default(x, 20)
    cv, neff, _ = krcv.kr_ll_cv_grid(x, y, h, k, with_neff=True)
    assert np.all(cv <= 1e-26), cv
    assert neff[-1] == 3000


@pytest.mark.parametrize("k", [U, E, T])
def test_ll_C2_full_size_sampled_shard(k):
    """Full C2 size (n = 20,000, 200 bandwidths) in the launch configuration
    the bench times: one sorted-order shard's S and n_eff row-exactly against
    the oracle; four shards add up to the whole search."""
    import torch
    x, y, h, _ = workloads.make("C2", seed=0)
    m = h.shape[0]
    d_x, d_y, d_h = (torch.as_tensor(a, device="cuda") for a in (x, y, h))
    ws = krcv.aligned(krcv.workspace(x.shape[0], m, "cuda"))
    part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device="cuda")
    krcv.kr_ll_shard_async(d_x, d_y, d_h, k, 41, 64, part, ws)
    torch.cuda.synchronize()
    p = part.cpu().numpy()
    ref = oracle.ll_cv(x, y, h, k, rows=oracle.shard_rows(x, 41, 64))
    assert cv_rel_err(p[:m], ref.S) <= TIGHT
    assert np.array_equal(p[m:2 * m].astype(np.int64), ref.neff)
    tot = np.zeros(krcv.partial_len(m))
    for r in range(4):
        krcv.kr_ll_shard_async(d_x, d_y, d_h, k, r, 4, part, ws)
        torch.cuda.synchronize()
        tot += part.cpu().numpy()
    cv, neff, best = krcv.kr_finalize(tot, x.shape[0], m)
    full, nfull, bfull = krcv.kr_ll_cv_grid(x, y, h, k, with_neff=True)
    assert cv_rel_err(cv, full) <= 1e-12 and np.array_equal(neff, nfull) and best == bfull


@pytest.mark.parametrize("shard", [0, 4095])
def test_ll_C5_full_size_tail_shards(shard):
    """Full C5 size (n = 200,000 lognormal x, 512 log-spaced bandwidths): the
    first and last sorted-order shards of 4,096 -- the sparse tails, where
    windows are small (direct branch) and rows drop out (M = 0)."""
    import torch
    x, y, h, k = workloads.make("C5", seed=0)
    m = h.shape[0]
    d_x, d_y, d_h = (torch.as_tensor(a, device="cuda") for a in (x, y, h))
    ws = krcv.aligned(krcv.workspace(x.shape[0], m, "cuda"))
    part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device="cuda")
    krcv.kr_ll_shard_async(d_x, d_y, d_h, k, shard, 4096, part, ws)
    torch.cuda.synchronize()
    p = part.cpu().numpy()
    ref = oracle.ll_cv(x, y, h, k, rows=oracle.shard_rows(x, shard, 4096))
    assert cv_rel_err(p[:m], ref.S) <= TIGHT
    assert np.array_equal(p[m:2 * m].astype(np.int64), ref.neff)


def test_ll_api_and_contract():
    """api.cv_grid(estimator="ll") = kr_ll_cv_grid bit for bit; deterministic;
    the Gaussian kernel is rejected (KR_EKERNEL)."""
    x, y = workloads.draw_xy("sin_uniform", 5000, 3)
    h = workloads.grid_default(x, 50)
    cv, best = krcv.kr_ll_cv_grid(x, y, h, E)
    r = cv_grid(x, y, h, kernel=E, estimator="ll")
    assert np.array_equal(r.cv.cpu().numpy(), cv) and r.best == best
    cv2, _ = krcv.kr_ll_cv_grid(x, y, h, E)
    assert np.array_equal(cv, cv2)
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_ll_cv_grid(x, y, h, GA)
    assert e.value.status == krcv.KR_EKERNEL
