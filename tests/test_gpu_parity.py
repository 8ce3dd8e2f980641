"""GPU parity: the CUDA path (through the C-ABI) vs the CPU oracle (T3, T4, T8).

Bar (BASELINE.json north_star): relative error <= 1e-6 on CV(h) with the
floor of SURVEY.md §8(c); n_eff identical; best identical unless the oracle's
two best values lie within 1e-6.  On well-conditioned workloads we also assert
a much tighter 1e-10 (fp64 vs long double is ~1e-14).
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
from oracle import exact
from paper_conf_ipps_rohlfsz17_b200 import krcv
from paper_conf_ipps_rohlfsz17_b200.api import GridSearch
from tests.helpers import best_ok, cv_rel_err

pytestmark = pytest.mark.gpu

U, E, T = 0, 1, 2
TOL = 1e-6
TIGHT = 1e-10
ALGO = {"a": "auto"}


@pytest.fixture(params=["sweep", "prefix"], autouse=True)
def algo(request):
    """Every parity test runs on both algorithms (KR_ALGO_SWEEP, KR_ALGO_PREFIX)."""
    ALGO["a"] = request.param
    yield request.param
    ALGO["a"] = "auto"


def _gpu(x, y, h, k):
    cv, neff, best = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo=ALGO["a"])
    return cv, neff, best


def _check(x, y, h, k, ref=None, tight=True):
    cv, neff, best = _gpu(x, y, h, k)
    if ref is None:
        ref = oracle.cv_sorted(x, y, h, k) if x.shape[0] > 400 else oracle.cv_direct(x, y, h, k)
    err = cv_rel_err(cv, ref.cv)
    assert err <= (TIGHT if tight else TOL), err
    assert np.array_equal(neff, ref.neff)
    assert best_ok(best, ref.cv), (best, ref.best)
    return err


@pytest.mark.parametrize("kname", ["epanechnikov", "uniform", "triangular"])
def test_worked_example_exact(kname):
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_example.json")))
    k = workloads.KERNEL_IDS[kname]
    cv, neff, best = _gpu(np.array(g["x"]), np.array(g["y"]), np.array(g["h"]), k)
    want = [float(Fraction(s)) for s in g[kname]["cv"]]
    for b in range(len(want)):
        assert abs(cv[b] - want[b]) <= 4 * math.ulp(want[b]) if want[b] else cv[b] == 0.0
    assert list(neff) == g[kname]["neff"] and best == g[kname]["best"]


@pytest.mark.parametrize("seed", range(16))
def test_exact_rational_dyadic(seed):
    """Dyadic inputs with points exactly at h and duplicated x: window
    membership must be bit-exact (n_eff identical), CV to fp64 rounding."""
    rng = np.random.default_rng(50 + seed)
    n = int(rng.integers(2, 17))
    m = int(rng.integers(1, 9))
    x, y, h = workloads.random_dyadic(n, m, seed)
    for k in (U, E, T):
        cv_ex, ne_ex, best_ex = exact.cv_exact(x, y, h, k)
        cv, neff, best = _gpu(x, y, h, k)
        assert cv_rel_err(cv, [float(v) for v in cv_ex]) <= 1e-13
        assert list(neff) == ne_ex
        assert best == best_ex or cv[best] == cv[best_ex]


@pytest.mark.parametrize("n", [2, 3, 31, 32, 33, 64, 65, 127, 1000])
@pytest.mark.parametrize("dist", ["paper", "sin_uniform", "lognormal"])
@pytest.mark.parametrize("k", [U, E, T])
def test_small_sizes_tiles_and_ragged_tails(n, dist, k):
    x, y = workloads.draw_xy(dist, n, 3)
    m = 37
    h = workloads.grid_log(x, m) if dist == "lognormal" else workloads.grid_default(x, m)
    _check(x, y, h, k)


@pytest.mark.parametrize("k", [U, E, T])
def test_user_grid_with_duplicates_and_small_h(k):
    x, y = workloads.draw_xy("paper", 777, 8)
    h = np.sort(np.concatenate([np.linspace(1e-4, 0.02, 20), [0.01, 0.01, 0.5, 0.5], np.linspace(0.3, 2.0, 9)]))
    _check(x, y, h, k)


@pytest.mark.parametrize("k", [U, E, T])
def test_duplicate_x_constant_y_and_equal_x(k):
    x, y = workloads.draw_xy("paper", 300, 9)
    x = np.round(x * 20) / 20  # heavy ties in x
    h = workloads.grid_default(x, 25)
    _check(x, y, h, k)
    cv, neff, best = _gpu(x, np.full_like(y, 4.0), h, k)
    assert np.all(cv == 0.0)
    # every x equal: all pairs at d = 0 -> g is the LOO mean
    xe = np.full(50, 0.75)
    ref = oracle.cv_direct(xe, y[:50], [0.1, 1.0], k)
    cv, neff, best = _gpu(xe, y[:50], np.array([0.1, 1.0]), k)
    assert cv_rel_err(cv, ref.cv) <= TIGHT and np.array_equal(neff, ref.neff)


@pytest.mark.parametrize("k", [E, T])
@pytest.mark.parametrize("yv", [(3.0, 5.0), (0.1, 7.0), (5.0, 0.125)])
def test_edge_cancellation_guard(k, yv):
    """One neighbour at d = nextafter(h, 0): guarded path returns g = y_l."""
    x = np.array([0.0, np.nextafter(1.0, 0.0)])
    y = np.array(yv)
    cv, neff, _ = _gpu(x, y, np.array([1.0]), k)
    want = float((Fraction(y[0]) - Fraction(y[1])) ** 2)
    assert abs(cv[0] - want) <= 2 * math.ulp(want) and neff[0] == 2


def test_boundary_exactly_at_h_uniform():
    """Default grid's last point h = r puts (min, max) exactly on the closed
    uniform window: GPU and oracle must agree bit-level on n_eff
    and the closed form."""
    x, y, h, k = workloads.make("C1", seed=0)
    _check(x, y, h, k)


def test_C1_seed0_full():
    x, y, h, k = workloads.make("C1", seed=0)
    cv, neff, best = _gpu(x, y, h, k)
    ref = oracle.cv_direct(x, y, h, k)
    assert cv_rel_err(cv, ref.cv) <= TIGHT and best == ref.best == 4


def test_C2_seed0_full():
    x, y, h, k = workloads.make("C2", seed=0)
    cv, neff, best = _gpu(x, y, h, k)
    ref = oracle.cv_sorted(x, y, h, k)
    assert cv_rel_err(cv, ref.cv) <= TIGHT
    assert np.array_equal(neff, ref.neff)
    assert best == ref.best == 1


def _device_partial(x, y, h, k, shard, nshards):
    import torch
    d_x = torch.as_tensor(x, device="cuda")
    d_y = torch.as_tensor(y, device="cuda")
    d_h = torch.as_tensor(h, device="cuda")
    part = torch.empty(krcv.partial_len(h.shape[0]), dtype=torch.float64, device="cuda")
    ws = krcv.aligned(krcv.workspace(x.shape[0], h.shape[0], "cuda"))
    krcv.kr_cv_shard_async(d_x, d_y, d_h, k, shard, nshards, part, ws, algo="auto" if k == 3 else ALGO["a"])
    torch.cuda.synchronize()
    return part.cpu().numpy()


@pytest.mark.parametrize("cfg,P,shard", [("C3", 64, 17), ("C5", 64, 0), ("C5", 64, 63), ("C4", 4096, 2048),
                                         ("C4", 4096, 40)])
def test_full_size_sampled_shard(cfg, P, shard):
    """Full BASELINE sizes in the bench launch configuration: one row shard of
    the sorted order, checked against the oracle on exactly those rows."""
    x, y, h, k = workloads.make(cfg, seed=0)
    part = _device_partial(x, y, h, k, shard, P)
    m = h.shape[0]
    ref = oracle.cv_sorted(x, y, h, k, rows=oracle.shard_rows(x, shard, P))
    assert cv_rel_err(part[:m], ref.S) <= TIGHT
    assert np.array_equal(part[m:2 * m].astype(np.int64), ref.neff)
    assert part[2 * m] == 0 and part[2 * m + 1] == 0


def test_row_ranges_sum_to_unsharded_and_match_oracle():
    """kr_cv_rows_async: disjoint unequal row ranges (incl. an empty one and
    ranges cutting through window-kernel tiles) add up to the unsharded
    partial, and one range equals the oracle on exactly those sorted rows."""
    import torch
    x, y, h, k = workloads.make("C5", seed=2, n=6000)
    m = h.shape[0]
    d_x, d_y, d_h = (torch.as_tensor(v, device="cuda") for v in (x, y, h))
    ws = krcv.aligned(krcv.workspace(x.shape[0], m, "cuda"))
    part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device="cuda")
    full = _device_partial(x, y, h, k, 0, 1)
    cuts = [0, 1, 777, 777, 2048, 4001, 5999, 6000]
    tot = np.zeros(krcv.partial_len(m))
    for lo, hi in zip(cuts, cuts[1:]):
        krcv.kr_cv_rows_async(d_x, d_y, d_h, k, lo, hi, part, ws, algo=ALGO["a"])
        torch.cuda.synchronize()
        p = part.cpu().numpy()
        tot += p
        if (lo, hi) == (777, 2048):
            ref = oracle.cv_sorted(x, y, h, k, rows=oracle.sorted_rows(x)[lo:hi])
            assert cv_rel_err(p[:m], ref.S) <= TIGHT
            assert np.array_equal(p[m:2 * m].astype(np.int64), ref.neff)
    assert cv_rel_err(tot[:m], full[:m]) <= 1e-14
    assert np.array_equal(tot[m:], full[m:])
    with pytest.raises(krcv.KrcvError):
        krcv.kr_cv_rows_async(d_x, d_y, d_h, k, 10, 5, part, ws)       # hi < lo
    with pytest.raises(krcv.KrcvError):
        krcv.kr_cv_rows_async(d_x, d_y, d_h, k, 0, 6001, part, ws)     # past n


@pytest.mark.parametrize("P", [2, 3, 8, 64])
def test_shard_emulation_sums_to_unsharded(P):
    """T4: shards 0..P-1 on one GPU, summed on the host == unsharded run."""
    x, y, h, k = workloads.make("C5", seed=1, n=5000)
    full = _device_partial(x, y, h, k, 0, 1)
    tot = sum(_device_partial(x, y, h, k, r, P) for r in range(P))
    m = h.shape[0]
    assert cv_rel_err(tot[:m], full[:m]) <= 1e-14
    assert np.array_equal(tot[m:], full[m:])
    cv, neff, best = krcv.kr_finalize(tot, x.shape[0], m)
    ref = oracle.cv_sorted(x, y, h, k)
    assert cv_rel_err(cv, ref.cv) <= TIGHT and best_ok(best, ref.cv)


def test_algorithms_agree():
    """Sweep and window-prefix give the same curve to ~1e-13 and identical
    n_eff (window membership is decided by the same binary64 predicate)."""
    for cfg, n in (("C2", 20000), ("C5", 20000), ("C1", 1000)):
        x, y, h, k = workloads.make(cfg, seed=4, n=n)
        a = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo="sweep")
        b = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo="prefix")
        assert cv_rel_err(b[0], a[0]) <= 1e-12
        assert np.array_equal(a[1], b[1]) and best_ok(b[2], a[0])


def test_determinism_bitwise():
    """T8: repeated runs are bit-identical (static row->warp map, fixed-order reductions)."""
    x, y, h, k = workloads.make("C2", seed=2, n=6000)
    a = _gpu(x, y, h, k)[0]
    for _ in range(3):
        assert np.array_equal(_gpu(x, y, h, k)[0], a)


def test_device_status_nonfinite_and_bad_grid():
    import torch
    x, y, h, k = workloads.make("C2", seed=0, n=500)
    x = x.copy()
    x[10] = np.nan
    part = _device_partial(x, y, h, k, 0, 1)
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_finalize(part, x.shape[0], h.shape[0])
    assert e.value.status == krcv.KR_ENONFINITE
    x[10] = 0.5
    hb = h.copy()
    hb[3] = -1.0
    part = _device_partial(x, y, hb, k, 0, 1)
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_finalize(part, x.shape[0], h.shape[0])
    assert e.value.status == krcv.KR_EGRID
    # device finalize reports the same status
    plan = GridSearch(x.shape[0], h, k, algo=ALGO["a"])
    xd = torch.as_tensor(x, device="cuda")
    yd = torch.as_tensor(y, device="cuda")
    xd[10] = float("inf")
    plan.run(xd, yd)
    with pytest.raises(krcv.KrcvError) as e:
        plan.result()
    assert e.value.status == krcv.KR_ENONFINITE


def test_device_api_matches_host_api():
    import torch
    x, y, h, k = workloads.make("C5", seed=0, n=20000)
    plan = GridSearch(x.shape[0], h, k, algo=ALGO["a"])
    plan.run(torch.as_tensor(x, device="cuda"), torch.as_tensor(y, device="cuda"))
    r = plan.result()
    cv, neff, best = _gpu(x, y, h, k)
    assert np.array_equal(r.cv.cpu().numpy(), cv)
    assert np.array_equal(r.neff.cpu().numpy(), neff) and r.best == best


def test_fused_finalize_matches_shard_plus_finalize():
    """kr_cv_grid_async (finalize fused into the reduction's last CTA) ==
    kr_cv_shard_async + host kr_finalize, bit for bit, over repeated calls
    (the completion counter must reset)."""
    import torch
    x, y, h, k = workloads.make("C5", seed=3, n=7000)
    part = _device_partial(x, y, h, k, 0, 1)
    cv0, ne0, b0 = krcv.kr_finalize(part, x.shape[0], h.shape[0])
    plan = GridSearch(x.shape[0], h, k, algo=ALGO["a"])
    xd, yd = torch.as_tensor(x, device="cuda"), torch.as_tensor(y, device="cuda")
    for _ in range(3):
        plan.run(xd, yd)
        r = plan.result()
        assert np.array_equal(r.cv.cpu().numpy(), cv0) and np.array_equal(r.neff.cpu().numpy(), ne0)
        assert r.best == b0


@pytest.mark.parametrize("m", [1, 2, 4099])
def test_grid_sizes(m):
    x, y = workloads.draw_xy("paper", 900, 1)
    h = workloads.grid_default(x, m)
    _check(x, y, h, E)


@pytest.mark.parametrize("k", [U, E, T])
def test_max_grid_size(k):
    """The largest grid the ABI accepts (KR_MAX_M = 65,536 bandwidths): tile
    partials, the reduction grid-stride loop and the fused finalize's arg-min
    at their limit, with a log grid so that windows range from empty to all."""
    x, y = workloads.draw_xy("lognormal", 300, 4)
    r = float(x.max() - x.min())
    h = np.geomspace(1e-6 * r, 2.0 * r, krcv.KR_MAX_M)
    cv, neff, best = _gpu(x, y, h, k)
    ref = oracle.cv_sorted(x, y, h, k)
    assert np.array_equal(neff, ref.neff)
    assert cv_rel_err(cv, ref.cv) <= TIGHT
    assert best_ok(best, ref.cv)


# The a2 implementations against each other (the library reads KRCV_SORT once
# per process, so that comparison runs in subprocesses):
# tests/test_gpu_sort_variants.py.


def test_rank_sort_heavy_duplicates():
    """Many equal x (ties broken by original index) through the rank sort."""
    x, y = workloads.draw_xy("paper", 9000, 2)
    x = np.floor(x * 7) / 7
    h = workloads.grid_default(x, 20)
    _check(x, y, h, E)


@pytest.mark.parametrize("k", [U, E, T])
@pytest.mark.parametrize("cfg", ["C2", "C5"])
def test_refine_matches_oracle(cfg, k):
    """kr_cv_refine (levels > 0 reuse the device-side sort / prefix moments,
    with grid sizes different from level 0) == the oracle's coarse-to-fine
    loop (oracle.cv_refine, reading Q22) level by level."""
    x, y, h, _ = workloads.make(cfg, seed=6, n=3000)
    hb, cb = krcv.kr_cv_refine(x, y, h, k, levels=4, m_fine=33, algo=ALGO["a"])
    hb_or, cb_or, _ = oracle.cv_refine(x, y, h, k, levels=4, m_fine=33)
    assert np.array_equal(hb, hb_or), (hb, hb_or)
    assert cv_rel_err(cb, cb_or) <= TIGHT
    with pytest.raises(krcv.KrcvError):
        krcv.kr_cv_refine(x, y, h, k, levels=3, m_fine=2)


# ---------------------------------------------------------------- Gaussian (dense path, Q23)
GA = 3


@pytest.mark.parametrize("n", [2, 33, 257, 1000])
@pytest.mark.parametrize("dist", ["paper", "sin_uniform", "lognormal"])
def test_gaussian_dense_parity(n, dist):
    """KR_GAUSSIAN through the tiled all-pairs kernel vs the oracle's direct
    long-double definition (with the Q23 rescaling); M_i = 1 for every row."""
    x, y = workloads.draw_xy(dist, n, 11)
    m = 21
    h = workloads.grid_log(x, m) if dist == "lognormal" else workloads.grid_default(x, m)
    cv, neff, best = krcv.kr_cv_grid(x, y, h, GA, with_neff=True)
    ref = oracle.cv_direct(x, y, h, GA)
    assert cv_rel_err(cv, ref.cv) <= TIGHT
    assert np.all(neff == n) and best_ok(best, ref.cv)


def test_gaussian_tiny_h_and_duplicates():
    """Bandwidths so small that unscaled weights would underflow fp64, and
    heavy ties in x (dmin = 0)."""
    x, y = workloads.draw_xy("paper", 600, 12)
    x = np.round(x * 50) / 50
    h = np.array([1e-5, 1e-3, 0.02, 0.3])
    cv, neff, best = krcv.kr_cv_grid(x, y, h, GA, with_neff=True)
    ref = oracle.cv_direct(x, y, h, GA)
    assert cv_rel_err(cv, ref.cv) <= TIGHT and np.all(neff == 600)


def test_gaussian_C2_sampled_shard():
    """Full C2 size (n = 20,000, 200 bandwidths) with the Gaussian kernel: one
    sorted-order shard checked row-exactly against the oracle."""
    x, y, h, _ = workloads.make("C2", seed=0)
    P, shard = 64, 21
    part = _device_partial(x, y, h, GA, shard, P)
    m = h.shape[0]
    ref = oracle.cv_direct(x, y, h, GA, rows=oracle.shard_rows(x, shard, P))
    assert cv_rel_err(part[:m], ref.S) <= TIGHT
    assert np.array_equal(part[m:2 * m].astype(np.int64), ref.neff)


def test_gaussian_algorithm_contract():
    x, y = workloads.draw_xy("paper", 100, 13)
    h = workloads.grid_default(x, 5)
    for a in ("sweep", "prefix"):
        with pytest.raises(krcv.KrcvError) as e:
            krcv.kr_cv_grid(x, y, h, GA, algo=a)
        assert e.value.status == krcv.KR_EARG
    with pytest.raises(krcv.KrcvError):
        krcv.kr_cv_grid(x, y, h, E, algo="dense")
    a = krcv.kr_cv_grid(x, y, h, GA, algo="dense")
    b = krcv.kr_cv_grid(x, y, h, GA)
    assert np.array_equal(a[0], b[0])


def test_gaussian_wide_bandwidth_chunk():
    """A chunk of bandwidths spanning more than 1e5 (the kernel's per-bandwidth
    clamp path) and the normal path give the oracle's curve."""
    x, y = workloads.draw_xy("lognormal", 700, 14)
    h = np.array([1e-7, 3e-6, 1e-4, 1e-2, 0.3, 2.0, 30.0, 200.0, 210.0])
    cv, neff, best = krcv.kr_cv_grid(x, y, h, GA, with_neff=True)
    ref = oracle.cv_direct(x, y, h, GA)
    assert cv_rel_err(cv, ref.cv) <= TIGHT and np.all(neff == 700)


# ---------------------------------------------------------------- KDE LSCV (Q24)
@pytest.mark.parametrize("k", [U, E, T])
@pytest.mark.parametrize("dist,n", [("paper", 2), ("paper", 65), ("paper", 1000), ("sin_uniform", 777),
                                    ("lognormal", 900)])
def test_kde_lscv_parity(k, dist, n):
    """kr_kde_lscv (window-prefix with u^1..u^5 dd prefix moments) vs the
    oracle's plain-definition KDE LSCV in long double."""
    x, _ = workloads.draw_xy(dist, n, 21)
    m = 31
    h = workloads.grid_log(x, m) if dist == "lognormal" else workloads.grid_default(x, m)
    lscv, best = krcv.kr_kde_lscv(x, h, k)
    ref = oracle.kde_lscv(x, h, k)
    assert cv_rel_err(lscv, ref.lscv) <= TIGHT
    assert best_ok(best, ref.lscv)


@pytest.mark.parametrize("k", [U, E, T])
def test_kde_full_size_sampled_shard(k):
    """C2-size x (n = 20,000, 200 bandwidths): one sorted-order shard's sums
    A and B against the oracle on exactly those rows; shards add up."""
    import torch
    x, _, h, _ = workloads.make("C2", seed=0)
    m = h.shape[0]
    d_x = torch.as_tensor(x, device="cuda")
    d_h = torch.as_tensor(h, device="cuda")
    ws = krcv.aligned(krcv.workspace(x.shape[0], m, "cuda"))
    part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device="cuda")
    krcv.kr_kde_shard_async(d_x, d_h, k, 37, 64, part, ws)
    torch.cuda.synchronize()
    p = part.cpu().numpy()
    ref = oracle.kde_lscv(x, h, k, rows=oracle.shard_rows(x, 37, 64))
    assert cv_rel_err(p[:m], ref.A) <= TIGHT and cv_rel_err(p[m:2 * m], ref.B) <= TIGHT
    tot = np.zeros(krcv.partial_len(m))
    for r in range(4):
        krcv.kr_kde_shard_async(d_x, d_h, k, r, 4, part, ws)
        torch.cuda.synchronize()
        tot += part.cpu().numpy()
    lscv, best = krcv.kr_kde_finalize(tot, x.shape[0], h, k)
    full, best_full = krcv.kr_kde_lscv(x, h, k)
    assert cv_rel_err(lscv, full) <= 1e-12 and best_ok(best, full)


def test_host_api_nonfinite_and_graph_replay():
    """kr_cv_grid from host arrays: NaN / Inf in x or y -> KR_ENONFINITE
    (device-side status) with the outputs untouched; with pinned buffers the
    call is replayed from a captured CUDA graph, which must read the buffers'
    current contents (new data each call) and re-capture when n, m, kernel
    or algorithm change."""
    import ctypes

    import torch
    lib = krcv._lib()
    x, y = workloads.draw_xy("paper", 3000, 5)
    h = workloads.grid_default(x, 40)
    for bad in ("x", "y"):
        xb, yb = x.copy(), y.copy()
        (xb if bad == "x" else yb)[1234] = math.nan if bad == "x" else -math.inf
        cv = np.full(40, 7.0)
        best = ctypes.c_int32(-5)
        st = lib.kr_cv_grid(xb.ctypes.data, yb.ctypes.data, 3000, h.ctypes.data, 40, E, cv.ctypes.data,
                            ctypes.byref(best))
        assert st == krcv.KR_ENONFINITE and np.all(cv == 7.0) and best.value == -5
    hx = torch.empty(3000, dtype=torch.float64).pin_memory()
    hy = torch.empty(3000, dtype=torch.float64).pin_memory()
    hh = torch.from_numpy(h.copy()).pin_memory()
    out = torch.empty(40, dtype=torch.float64).pin_memory()
    best = ctypes.c_int32(-1)
    for seed in range(4):
        xs, ys = workloads.draw_xy("sin_uniform" if seed % 2 else "paper", 3000, 50 + seed)
        hx.copy_(torch.from_numpy(xs))
        hy.copy_(torch.from_numpy(ys))
        hh.copy_(torch.from_numpy(workloads.grid_default(xs, 40)))
        for k in (E, U):
            st = krcv.kr_cv_grid_ptr(hx.data_ptr(), hy.data_ptr(), 3000, hh.data_ptr(), 40, k, out.data_ptr(),
                                     ctypes.byref(best))
            assert st == 0
            ref = oracle.cv_sorted(xs, ys, hh.numpy(), k)
            assert cv_rel_err(out.numpy(), ref.cv) <= TIGHT and best.value == ref.best
    # a NaN arriving through the replayed graph is still reported
    hx[7] = math.nan
    st = krcv.kr_cv_grid_ptr(hx.data_ptr(), hy.data_ptr(), 3000, hh.data_ptr(), 40, U, out.data_ptr(),
                             ctypes.byref(best))
    assert st == krcv.KR_ENONFINITE


def test_gridsearch_graph_replay():
    """GridSearch(graph=True): the captured graph replays the whole search;
    new contents in the same tensors are picked up, other tensors re-capture,
    results equal the eager path bit for bit (same kernels, same order)."""
    import torch
    x, y = workloads.draw_xy("paper", 5000, 9)
    h = workloads.grid_default(x, 60)
    d_x, d_y = torch.as_tensor(x, device="cuda"), torch.as_tensor(y, device="cuda")
    eager = GridSearch(5000, h, E)
    graph = GridSearch(5000, h, E, graph=True)
    for step in range(3):
        if step == 2:
            d_x, d_y = d_x.clone(), (d_y * 2.0).contiguous()
        elif step == 1:
            d_y.mul_(0.5)
        eager.run(d_x, d_y)
        graph.run(d_x, d_y)
        a, b = eager.result(), graph.result()
        assert torch.equal(a.cv, b.cv) and a.best == b.best and torch.equal(a.neff, b.neff)
    ref = oracle.cv_sorted(d_x.cpu().numpy(), d_y.cpu().numpy(), h, E)
    assert cv_rel_err(b.cv.cpu().numpy(), ref.cv) <= TIGHT


def test_gridsearch_graph_with_stage_events():
    """The bench's configuration: profiling on before the capture, so the
    stage events are event-record nodes of the graph and kr_profile_read
    returns this replay's stage times."""
    import torch
    x, y, h, k = workloads.make("C2", seed=0, n=4000)
    d_x, d_y = torch.as_tensor(x, device="cuda"), torch.as_tensor(y, device="cuda")
    krcv.kr_profile_enable(True)
    try:
        plan = GridSearch(4000, h, k, graph=True)
        for _ in range(3):
            plan.run(d_x, d_y)
            st = krcv.kr_profile_read()
            assert len(st) == 4 and all(v >= 0.0 for v in st) and st[2] > 0.0
    finally:
        krcv.kr_profile_enable(False)
    ref = oracle.cv_sorted(x, y, h, k)
    assert cv_rel_err(plan.result().cv.cpu().numpy(), ref.cv) <= TIGHT
