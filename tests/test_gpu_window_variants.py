"""GPU: the window-kernel variants find the same boundaries.

`window_kernel_blk` (KRCV_WIN_K = 9 / 10: 2 / 4 blocks of 32 consecutive rows)
sums a tile's rows in another order than window_kernel<K, 2 / 4>: n_eff and
best must be identical, CV equal to rounding.

`window_kernel_seg` (KRCV_WIN_K = 6 / 7 / 8: 2 / 4 / 1 rows per lane) searches
in a shared-memory segment with an exact check of its prediction and falls
back to `window_kernel`'s global searches; with the same rows per lane
(KRCV_WIN_K = 2 / 4 / 1) the two kernels group rows into the same tiles, so
their CV curves must agree bit for bit.  The library reads KRCV_WIN_K once per
process, so each variant runs in a subprocess.  Inputs stress the fallback:
heavy-tailed x (sparse tiles, segments longer than the cap), duplicates,
points exactly at a bandwidth, a jump in the grid, tiny n.
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
    return cases


def _run(k: int, path: str):
    env = dict(os.environ, KRCV_WIN_K=str(k))
    p = subprocess.run([sys.executable, "-c", CHILD, path], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=600)
    assert p.returncode == 0, p.stderr[-2000:]
    return json.loads(p.stdout.strip().splitlines()[-1])


@pytest.mark.parametrize("base,seg", [(2, 6), (4, 7), (1, 8)])
def test_seg_kernel_bit_identical(tmp_path, base, seg):
    cases = _cases()
    path = str(tmp_path / "cases.npz")
    arrs = {}
    for c, (x, y, h, k) in cases.items():
        arrs[c + "_x"], arrs[c + "_y"], arrs[c + "_h"], arrs[c + "_k"] = x, y, h, np.array(k)
    np.savez(path, **arrs)
    a, b = _run(base, path), _run(seg, path)
    for c in cases:
        assert a[c]["cv"] == b[c]["cv"], c
        assert a[c]["neff"] == b[c]["neff"], c
        assert a[c]["best"] == b[c]["best"], c


@pytest.mark.parametrize("base,blk", [(2, 9), (4, 10)])
def test_blk_kernel_same_windows(tmp_path, base, blk):
    cases = _cases()
    path = str(tmp_path / "cases.npz")
    arrs = {}
    for c, (x, y, h, k) in cases.items():
        arrs[c + "_x"], arrs[c + "_y"], arrs[c + "_h"], arrs[c + "_k"] = x, y, h, np.array(k)
    np.savez(path, **arrs)
    a, b = _run(base, path), _run(blk, path)
    for c in cases:
        ca = np.array(a[c]["cv"], np.uint64).view(np.float64)
        cb = np.array(b[c]["cv"], np.uint64).view(np.float64)
        assert a[c]["neff"] == b[c]["neff"], c
        scale = max(float(np.max(np.abs(ca))), 1e-300)
        assert float(np.max(np.abs(ca - cb))) <= 1e-13 * scale, c
        assert a[c]["best"] == b[c]["best"], c
