"""GPU: the anchored fast-path records (anchor_kernel).

win_kernel's Epanechnikov fast path reads J copies of the prefix hi words
anchored at the centres of J index regions (krcv_window.cuh); the library
uses them from n = 50,000 on, so the small parity cases elsewhere never reach
them.  Here every J (KRCV_ANCHORS, read once per process: one subprocess per
J) runs the window-variant stress inputs -- heavy tail, duplicates, points
exactly at a bandwidth, a jump in the grid, tiny n, all x equal, two values --
plus a paper-DGP case at n = 50,000 that the default rule anchors, against
Program 3 (oracle.cv_sorted): the windows (n_eff) exactly, the curve to the
bar the other window tests use, and the anchored curve against the
unanchored one (J = 0) to rounding.
"""
from __future__ import annotations

import numpy as np
import pytest

from tests.test_gpu_window_variants import _cases, _run

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def anchor_cases(tmp_path_factory):
    cases = {k: v for k, v in _cases().items() if v[3] == "epanechnikov"}
    rng = np.random.default_rng(11)
    x = rng.uniform(0, 1, 50000)
    y = 0.5 * x + 10 * x * x + rng.uniform(0, 0.5, 50000)
    cases["paper50k"] = (x, y, np.geomspace(2e-5, 1.0, 24), "epanechnikov")
    xs = rng.uniform(-3, 5, 9000)
    cases["shifted"] = (xs, np.cos(xs) + rng.normal(0, 0.1, 9000), np.geomspace(1e-4, 8.0, 48), "epanechnikov")
    path = str(tmp_path_factory.mktemp("anchors") / "cases.npz")
    arrs = {}
    for c, (x, y, h, k) in cases.items():
        arrs[c + "_x"], arrs[c + "_y"], arrs[c + "_h"], arrs[c + "_k"] = x, y, h, np.array(k)
    np.savez(path, **arrs)
    return path, cases


@pytest.fixture(scope="module")
def unanchored(anchor_cases):
    return _run({"KRCV_ANCHORS": "0"}, anchor_cases[0])


@pytest.fixture(scope="module")
def refs(anchor_cases):
    import oracle

    return {c: oracle.cv_sorted(x, y, h, 1) for c, (x, y, h, _) in anchor_cases[1].items()}


@pytest.mark.parametrize("J", ["1", "3", "8", "16", "default"])
def test_anchored_matches_oracle_and_unanchored(anchor_cases, unanchored, refs, J):
    from tests.helpers import best_ok, cv_rel_err

    path, cases = anchor_cases
    a = _run({} if J == "default" else {"KRCV_ANCHORS": J}, path)
    for c in cases:
        ref = refs[c]
        got = np.array(a[c]["cv"], np.uint64).view(np.float64)
        assert cv_rel_err(got, ref.cv) <= 1e-10, (c, J)
        assert np.array_equal(np.asarray(a[c]["neff"]), ref.neff), (c, J)
        assert best_ok(a[c]["best"], ref.cv), (c, J)
        base = np.array(unanchored[c]["cv"], np.uint64).view(np.float64)
        scale = max(float(np.max(np.abs(base))), 1e-300)
        assert float(np.max(np.abs(got - base))) <= 1e-13 * scale, (c, J)


def test_anchored_row_ranges_sum_to_unsharded():
    """A row range builds only the anchored copies of its rows' regions (DESIGN.md
    §6.2) and clamps every task's anchor to them: disjoint ranges -- cutting
    through anchor regions (n / 8 = 7,500 rows here), ending one and two rows
    past a region boundary, spanning several regions, empty -- on one reused
    workspace add up to the unsharded partial (windows exactly, sums to
    rounding), and one range equals Program 3 on exactly those sorted rows."""
    import torch

    import oracle
    import workloads
    from paper_conf_ipps_rohlfsz17_b200 import krcv
    from tests.helpers import cv_rel_err

    x, y, h, k = workloads.make("C5", seed=4, n=60000)
    h = h[::8].copy()
    m = h.shape[0]
    d_x, d_y, d_h = (torch.as_tensor(v, device="cuda") for v in (x, y, h))
    ws = krcv.aligned(krcv.workspace(x.shape[0], m, "cuda"))
    part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device="cuda")
    krcv.kr_cv_rows_async(d_x, d_y, d_h, k, 0, 60000, part, ws)
    torch.cuda.synchronize()
    full = part.cpu().numpy().copy()
    cuts = [0, 7490, 7501, 7502, 7502, 22500, 22530, 51000, 59999, 60000]
    tot = np.zeros(krcv.partial_len(m))
    for lo, hi in zip(cuts, cuts[1:]):
        krcv.kr_cv_rows_async(d_x, d_y, d_h, k, lo, hi, part, ws)
        torch.cuda.synchronize()
        p = part.cpu().numpy()
        tot += p
        if (lo, hi) == (7490, 7501):
            ref = oracle.cv_sorted(x, y, h, k, rows=oracle.sorted_rows(x)[lo:hi])
            assert cv_rel_err(p[:m], ref.S) <= 1e-10
            assert np.array_equal(p[m:2 * m].astype(np.int64), ref.neff)
    assert cv_rel_err(tot[:m], full[:m]) <= 1e-13
    assert np.array_equal(tot[m:], full[m:])
