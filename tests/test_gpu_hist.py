"""GPU parity of the histogram ordering (KR_ALGO_HIST, krcv_hist.cuh; SURVEY.md
§7.1 design "H", the north_star's "bucket-by-bandwidth shared-memory
histogram followed by a warp-shuffle scan") through the C-ABI vs the oracle.

The shared-memory atomics make the summation order timing-dependent, so the
bar is the tolerance (1e-10 on these workloads, north_star 1e-6), n_eff exact
(integer work) and best by the tie rule -- not bitwise equality.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import workloads
from paper_conf_ipps_rohlfsz17_b200 import krcv
from tests.helpers import best_ok, cv_rel_err

pytestmark = pytest.mark.gpu

U, E, T, GA = 0, 1, 2, 3
TIGHT = 1e-10


def _check(x, y, h, k):
    cv, neff, best = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo="hist")
    ref = oracle.cv_sorted(x, y, h, k) if x.shape[0] > 400 else oracle.cv_direct(x, y, h, k)
    assert cv_rel_err(cv, ref.cv) <= TIGHT
    assert np.array_equal(neff, ref.neff)
    assert best_ok(best, ref.cv)


@pytest.mark.parametrize("k", [U, E, T])
@pytest.mark.parametrize("dist,n", [("paper", 2), ("paper", 33), ("paper", 257), ("sin_uniform", 1000),
                                    ("lognormal", 900)])
def test_hist_parity(k, dist, n):
    x, y = workloads.draw_xy(dist, n, 17)
    m = 41
    h = workloads.grid_log(x, m) if dist == "lognormal" else workloads.grid_default(x, m)
    _check(x, y, h, k)


@pytest.mark.parametrize("k", [U, E, T])
def test_hist_dyadic_duplicates_edges(k):
    """Points exactly at h (bucket boundaries decided by the exact predicate),
    duplicate x (d = 0 neighbours go to bucket 0)."""
    for seed in range(8):
        x, y, h = workloads.random_dyadic(int(np.random.default_rng(seed).integers(2, 60)), 6, 300 + seed)
        _check(x, y, h, k)


@pytest.mark.parametrize("k", [U, E])
def test_hist_C2_full_size_sampled_shard(k):
    """Full C2 size in the launch configuration: one sorted-order shard's S and
    n_eff row-exactly against the oracle."""
    import torch
    x, y, h, _ = workloads.make("C2", seed=0)
    m = h.shape[0]
    d_x, d_y, d_h = (torch.as_tensor(a, device="cuda") for a in (x, y, h))
    ws = krcv.aligned(krcv.workspace(x.shape[0], m, "cuda"))
    part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device="cuda")
    krcv.kr_cv_shard_async(d_x, d_y, d_h, k, 9, 64, part, ws, algo="hist")
    torch.cuda.synchronize()
    p = part.cpu().numpy()
    ref = oracle.cv_sorted(x, y, h, k, rows=oracle.shard_rows(x, 9, 64))
    assert cv_rel_err(p[:m], ref.S) <= TIGHT
    assert np.array_equal(p[m:2 * m].astype(np.int64), ref.neff)


@pytest.mark.parametrize("k", [U, E, T])
def test_hist_grid_size_limits(k):
    """m = 4,099 runs in one shared-memory histogram with one warp per CTA;
    m = 6,000 and 12,345 do not fit one and run as slices of the grid (a
    bucket is the first bandwidth of the slice whose window holds the
    neighbour, so each slice's running sums are the full grid's); the
    Gaussian kernel is rejected."""
    x, y = workloads.draw_xy("paper", 300, 2)
    _check(x, y, workloads.grid_default(x, 4099), k)
    _check(x, y, workloads.grid_default(x, 6000), k)
    r = float(x.max() - x.min())
    _check(x, y, np.geomspace(1e-4 * r, 2.0 * r, 12345), k)
    with pytest.raises(krcv.KrcvError) as e:
        krcv.kr_cv_grid(x, y, workloads.grid_default(x, 10), GA, algo="hist")
    assert e.value.status == krcv.KR_EARG
