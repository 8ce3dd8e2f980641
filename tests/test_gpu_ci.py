"""GPU parity of the leave-one-out (delete-one jackknife) confidence intervals
at the cross-validated bandwidth (PAPER.md P@10560, SURVEY §8(f) rank 3,
reading Q26; krcv_ci.cuh) against the oracle's plain definitions
(oracle.cv_ci / oracle.kde_ci, long double; themselves pinned by the
jackknife computed by explicit deletion in exact rationals,
tests/test_oracle_pins.py P12).

Element by element: the optimal index, est[n] and se[n] to 1e-10 relative
(floor: the scale of the estimates), NaN exactly where the oracle has no
interval (a window holding only its point).  Sizes from n = 2 to a full-size
C2 problem; uniform / heavy-tailed / dyadic-tied x; all three compact kernels;
the device entry points and the host ones give the same result."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu

TOL = 1e-10
KERNELS = {"uniform": 0, "epanechnikov": 1, "triangular": 2}


def _rel(got, ref, floor):
    got, ref = np.asarray(got, np.float64), np.asarray(ref, np.float64)
    nan_g, nan_r = np.isnan(got), np.isnan(ref)
    assert np.array_equal(nan_g, nan_r), (np.flatnonzero(nan_g != nan_r)[:10])
    ok = ~nan_r
    if not ok.any():
        return 0.0
    return float(np.max(np.abs(got[ok] - ref[ok]) / np.maximum(np.abs(ref[ok]), floor)))


def _cases():
    out = []
    for n in (2, 3, 37, 500, 3001):
        for dist in ("paper", "lognormal"):
            x, y = workloads.draw_xy(dist, n, 11 + n)
            r = float(x.max() - x.min())
            h = np.geomspace(1e-3 * r, r, 24) if dist == "lognormal" else workloads.grid_default(x, 30)
            out.append((f"{dist}-{n}", x, y, h))
    rng = np.random.default_rng(2)
    xd = np.floor(rng.uniform(0, 64, 700)) / 16.0  # ties and pairs exactly at h
    yd = rng.normal(0, 1, 700)
    out.append(("dyadic", xd, yd, np.concatenate([np.arange(1, 17) / 16.0, [2.0, 4.0]])))
    return out


CASES = _cases()


@pytest.mark.parametrize("kname", list(KERNELS))
@pytest.mark.parametrize("case", CASES, ids=[c[0] for c in CASES])
def test_nw_ci_matches_oracle(case, kname):
    from paper_conf_ipps_rohlfsz17_b200 import krcv

    _, x, y, h = case
    k = KERNELS[kname]
    cv, est, se, best = krcv.kr_cv_ci(x, y, h, kname)
    ref = oracle.cv_ci(x, y, h, k)
    assert best == ref.best
    scale = float(np.max(np.abs(y)))
    assert _rel(est, ref.est, 1e-12 * scale) <= TOL
    assert _rel(se, ref.se, 1e-12 * scale) <= TOL


@pytest.mark.parametrize("kname", list(KERNELS))
@pytest.mark.parametrize("case", CASES, ids=[c[0] for c in CASES])
def test_kde_ci_matches_oracle(case, kname):
    from paper_conf_ipps_rohlfsz17_b200 import krcv

    _, x, _, h = case
    k = KERNELS[kname]
    lscv, est, se, best = krcv.kr_kde_ci(x, h, kname)
    ref = oracle.kde_ci(x, h, k)
    assert best == ref.best
    scale = float(np.max(ref.est))
    assert _rel(est, ref.est, 1e-12 * scale) <= TOL
    assert _rel(se, ref.se, 1e-12 * scale) <= TOL


def test_ci_full_size_c2_and_device_entry_points():
    """C2 in full (n = 20,000, Epanechnikov, the bench's config) through the
    device entry points -- against the oracle and bit-identical to the host
    entry point -- and the interval helper."""
    import torch

    from paper_conf_ipps_rohlfsz17_b200 import krcv

    x, y, h, k = workloads.make("C2", seed=0)
    n, m = x.shape[0], h.shape[0]
    dev = torch.device("cuda", 0)
    d_x, d_y, d_h = (torch.as_tensor(a, device=dev) for a in (x, y, h))
    ws = krcv.aligned(krcv.workspace(n, m, dev))
    d_cv = torch.empty(m, dtype=torch.float64, device=dev)
    d_est = torch.empty(n, dtype=torch.float64, device=dev)
    d_se = torch.empty(n, dtype=torch.float64, device=dev)
    bs = torch.empty(2, dtype=torch.int32, device=dev)
    krcv.kr_cv_ci_async(d_x, d_y, d_h, k, d_cv, d_est, d_se, bs, ws)
    torch.cuda.synchronize()
    assert int(bs[1]) == 0
    ref = oracle.cv_ci(x, y, h, k)
    assert int(bs[0]) == ref.best == 1  # C2 seed 0 optimum b = 1
    assert _rel(d_est.cpu().numpy(), ref.est, 1e-12) <= TOL
    assert _rel(d_se.cpu().numpy(), ref.se, 1e-12) <= TOL
    cv, est, se, best = krcv.kr_cv_ci(x, y, h, k)
    assert best == ref.best
    assert np.array_equal(est, d_est.cpu().numpy()) and np.array_equal(se, d_se.cpu().numpy())
    lo, hi = krcv.confidence_intervals(est, se, 0.95)
    assert np.all(lo <= est) and np.all(est <= hi)
    # KDE on the same x, device form (the first 6 bandwidths: the oracle's
    # LSCV is the O(n^2 m) plain definition)
    hk = h[:6]
    d_hk = torch.as_tensor(hk, device=dev)
    d_l = torch.empty(hk.shape[0], dtype=torch.float64, device=dev)
    krcv.kr_kde_ci_async(d_x, d_hk, k, d_l, d_est, d_se, bs, ws)
    torch.cuda.synchronize()
    rk = oracle.kde_ci(x, hk, k)
    assert int(bs[0]) == rk.best
    assert _rel(d_est.cpu().numpy(), rk.est, 1e-12) <= TOL
    assert _rel(d_se.cpu().numpy(), rk.se, 1e-12) <= TOL


def test_ci_rejects_gaussian_and_bad_grid():
    from paper_conf_ipps_rohlfsz17_b200 import krcv

    x, y, h, _ = workloads.make("C1", seed=0, n=100)
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_cv_ci(x, y, h, "gaussian")
    assert e.value.status == krcv.KR_EKERNEL
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_cv_ci(x, y, h[::-1], "epanechnikov")
    assert e.value.status == krcv.KR_EGRID
