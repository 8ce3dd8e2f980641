"""GPU: the window kernels find the same boundaries.

`win_kernel` (krcv_window.cuh, the default) looks every boundary up in a
bucket table and verifies it with the exact binary64 predicate of reading Q1;
r01's `window_kernel<K>` / `window_kernel_b2` (KRCV_WIN=r01, KRCV_WIN_K = 1 /
2 / 3) search from the previous bandwidth's boundaries.  The windows -- hence
n_eff -- must be identical, and so must best; the CV curves are equal to
rounding (the kernels sum a bandwidth's squared errors in different orders:
one partial per 32-row tile vs per block of tiles).  The library reads the
selection once per process, so each variant runs in a subprocess.  Inputs
stress the lookups: heavy-tailed x (crowded and empty buckets, F at its cap),
duplicates, points exactly at a bandwidth, a jump in the grid, tiny n, all x
equal (zero span), two distinct values.
"""
from __future__ import annotations

import json
import os
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, sys
import numpy as np
from paper_conf_ipps_rohlfsz17_b200 import krcv
d = np.load(sys.argv[1])
out = {}
for name in d.files:
    if not name.endswith("_x"):
        continue
    c = name[:-2]
    x, y, h, k = d[c + "_x"], d[c + "_y"], d[c + "_h"], str(d[c + "_k"])
    cv, neff, best = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo="prefix")
    out[c] = {"cv": np.asarray(cv, np.float64).view(np.uint64).tolist(), "neff": np.asarray(neff).tolist(), "best": int(best)}
print(json.dumps(out))
"""


def _cases():
    rng = np.random.default_rng(7)
    cases = {}
    n = 30000
    x = rng.lognormal(0.0, 1.0, n)
    y = np.sin(x) + rng.normal(0, 0.5, n)
    r = x.max() - x.min()
    cases["lognormal"] = (x, y, np.geomspace(1e-4 * r, r, 96), "epanechnikov")
    cases["lognormal_u"] = (x, y, np.geomspace(1e-4 * r, r, 64), "uniform")
    x = rng.uniform(0, 1, 20000)
    y = 0.5 * x + 10 * x * x + rng.uniform(0, 0.5, 20000)
    cases["paper"] = (x, y, np.arange(1, 121) / 120.0, "epanechnikov")
    cases["paper_t"] = (x, y, np.arange(1, 81) / 80.0, "triangular")
    # dyadic grid points and duplicates: many pairs exactly at a bandwidth
    xd = np.floor(rng.uniform(0, 256, 5000)) / 64.0
    yd = rng.normal(0, 1, 5000)
    hd = np.concatenate([np.arange(1, 40) / 64.0, [1.0, 3.0, 3.0, 4.0]])
    cases["dyadic_u"] = (xd, yd, hd, "uniform")
    cases["dyadic_e"] = (xd, yd, hd, "epanechnikov")
    # jump in the grid (growth prediction far off), tiny n
    xs = rng.uniform(0, 1, 3000)
    ys = rng.normal(0, 1, 3000)
    hj = np.concatenate([np.linspace(1e-4, 1e-3, 20), np.linspace(0.2, 1.0, 20)])
    cases["jump"] = (xs, ys, hj, "epanechnikov")
    cases["tiny"] = (xs[:37], ys[:37], np.linspace(0.01, 1.0, 30), "epanechnikov")
    cases["const_x"] = (np.full(300, 0.5), ys[:300], np.array([1e-3, 0.1, 1.0]), "epanechnikov")
    cases["two_values"] = (np.repeat([0.0, 1.0], 150), ys[:300], np.array([0.5, 1.0, 1.0, 2.0]), "uniform")
    return cases


def _run(env_extra: dict, path: str):
    env = dict(os.environ, **env_extra)
    p = subprocess.run([sys.executable, "-c", CHILD, path], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=600)
    assert p.returncode == 0, p.stderr[-2000:]
    return json.loads(p.stdout.strip().splitlines()[-1])


@pytest.fixture(scope="module")
def case_path(tmp_path_factory):
    cases = _cases()
    path = str(tmp_path_factory.mktemp("winvar") / "cases.npz")
    arrs = {}
    for c, (x, y, h, k) in cases.items():
        arrs[c + "_x"], arrs[c + "_y"], arrs[c + "_h"], arrs[c + "_k"] = x, y, h, np.array(k)
    np.savez(path, **arrs)
    return path, cases


@pytest.mark.parametrize("r01k", ["1", "2", "3"])
def test_win_kernel_same_windows_as_r01(case_path, r01k):
    path, cases = case_path
    a = _run({}, path)
    b = _run({"KRCV_WIN": "r01", "KRCV_WIN_K": r01k}, path)
    for c in cases:
        ca = np.array(a[c]["cv"], np.uint64).view(np.float64)
        cb = np.array(b[c]["cv"], np.uint64).view(np.float64)
        assert a[c]["neff"] == b[c]["neff"], c
        scale = max(float(np.max(np.abs(ca))), 1e-300)
        assert float(np.max(np.abs(ca - cb))) <= 1e-13 * scale, c
        assert a[c]["best"] == b[c]["best"], c


def test_win_kernel_matches_oracle(case_path):
    """The default kernel on the same stress inputs against Program 3."""
    import oracle
    from tests.helpers import best_ok, cv_rel_err

    path, cases = case_path
    a = _run({}, path)
    kid = {"uniform": 0, "epanechnikov": 1, "triangular": 2}
    for c, (x, y, h, k) in cases.items():
        ref = oracle.cv_sorted(x, y, h, kid[k])
        got = np.array(a[c]["cv"], np.uint64).view(np.float64)
        assert cv_rel_err(got, ref.cv) <= 1e-10, c
        assert np.array_equal(np.asarray(a[c]["neff"]), ref.neff), c
        assert best_ok(a[c]["best"], ref.cv), c
