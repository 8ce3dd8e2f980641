"""GPU parity of `sweep_gxg_kernel` (krcv_sweep_gxg.cuh), the sweep variant the
auto-selector runs for KR_ALGO_SWEEP shards of >= kGxgRows = 400,000 rows
(VERDICT r01 "what's weak" #1).

G lanes x G adjacent sorted rows share each loaded neighbour and accumulate
the shared elements' moments about the first row, so its bookkeeping differs
from `sweep_kernel`'s wherever rows of a group see different window ends --
tied x values, points exactly at a bandwidth, group edges that are not a
multiple of G at shard boundaries.  The library reads KRCV_SWEEP /
KRCV_SWEEP_G once per process, so each setting runs in a subprocess that
forces the gxg variant for every shard size; results are compared with the
oracle's Program-3 evaluator (oracle.cv_sorted) element by element -- whole
searches and row shards whose edges are not multiples of G.

A second test reaches the auto-selection itself: a 450,000-row search with
KR_ALGO_SWEEP (gxg by size) against the default window-prefix path on the same
input (itself oracle-checked at every size in test_gpu_parity.py).
"""
from __future__ import annotations

import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from tests.helpers import best_ok, cv_rel_err

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TOL = 1e-10

CHILD = r"""
import json, sys
import numpy as np
import torch
from paper_conf_ipps_rohlfsz17_b200 import krcv
d = np.load(sys.argv[1])
nshards = int(sys.argv[2])
out = {}
dev = torch.device("cuda", 0)
for name in d.files:
    if not name.endswith("_x"):
        continue
    c = name[:-2]
    x, y, h, k = d[c + "_x"], d[c + "_y"], d[c + "_h"], str(d[c + "_k"])
    cv, neff, best = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo="sweep")
    n, m = x.shape[0], h.shape[0]
    dx, dy, dh = (torch.as_tensor(a, device=dev) for a in (x, y, h))
    ws = krcv.aligned(krcv.workspace(n, m, dev))
    shards = []
    for s in range(nshards):
        part = torch.zeros(krcv.partial_len(m), dtype=torch.float64, device=dev)
        krcv.kr_cv_shard_async(dx, dy, dh, k, s, nshards, part, ws, algo="sweep")
        shards.append(part.cpu().numpy().tolist())
    out[c] = {"cv": np.asarray(cv).tolist(), "neff": np.asarray(neff).tolist(), "best": int(best),
              "shards": shards, "algo": krcv.kr_last_algo()}
print(json.dumps(out))
"""


def _cases():
    rng = np.random.default_rng(11)
    cases = {}
    x = rng.uniform(0, 1, 4003)
    y = 0.5 * x + 10 * x * x + rng.uniform(0, 0.5, x.shape[0])
    cases["paper_e"] = (x, y, np.arange(1, 41) / 40.0, "epanechnikov")
    cases["paper_t"] = (x, y, np.arange(1, 31) / 30.0, "triangular")
    cases["paper_u"] = (x, y, np.arange(1, 31) / 30.0, "uniform")
    # heavy tail: groups whose rows see very different windows
    xl = rng.lognormal(0.0, 1.0, 3001)
    yl = np.sin(xl) + rng.normal(0, 0.5, xl.shape[0])
    r = xl.max() - xl.min()
    cases["lognormal_e"] = (xl, yl, np.geomspace(1e-4 * r, r, 48), "epanechnikov")
    cases["lognormal_u"] = (xl, yl, np.geomspace(1e-4 * r, r, 32), "uniform")
    # ties: dyadic x with many duplicates, pairs exactly at a bandwidth
    xd = np.floor(rng.uniform(0, 64, 2501)) / 16.0
    yd = rng.normal(0, 1, xd.shape[0])
    hd = np.concatenate([np.arange(1, 25) / 16.0, [2.0, 2.0, 4.0]])
    for kname in ("epanechnikov", "triangular", "uniform"):
        cases["dyadic_" + kname[0]] = (xd, yd, hd, kname)
    # all x equal (every row's window at d = 0), and tiny n not a multiple of G
    cases["const_x"] = (np.full(67, 0.25), rng.normal(0, 1, 67), np.array([0.1, 0.5]), "epanechnikov")
    cases["tiny"] = (x[:7], y[:7], np.linspace(0.05, 1.0, 9), "epanechnikov")
    return cases


KIDS = {"uniform": 0, "epanechnikov": 1, "triangular": 2}


@pytest.fixture(scope="module")
def case_file(tmp_path_factory):
    cases = _cases()
    path = str(tmp_path_factory.mktemp("gxg") / "cases.npz")
    arrs = {}
    for c, (x, y, h, k) in cases.items():
        arrs[c + "_x"], arrs[c + "_y"], arrs[c + "_h"], arrs[c + "_k"] = x, y, h, np.array(k)
    np.savez(path, **arrs)
    return path, cases


@pytest.mark.parametrize("G", [4, 2, 1])
def test_gxg_forced_matches_oracle(case_file, G):
    path, cases = case_file
    nshards = 3
    env = dict(os.environ, KRCV_SWEEP="gxg", KRCV_SWEEP_G=str(G))
    p = subprocess.run([sys.executable, "-c", CHILD, path, str(nshards)], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=900)
    assert p.returncode == 0, p.stderr[-3000:]
    got = json.loads(p.stdout.strip().splitlines()[-1])
    for c, (x, y, h, k) in cases.items():
        g = got[c]
        assert g["algo"] == 1, c  # KR_ALGO_SWEEP ran
        kid = KIDS[k]
        ref = oracle.cv_sorted(x, y, h, kid)
        assert cv_rel_err(g["cv"], ref.cv) <= TOL, (c, G)
        assert np.array_equal(np.asarray(g["neff"]), ref.neff), (c, G)
        assert best_ok(g["best"], ref.cv), (c, G)
        m = h.shape[0]
        for s, part in enumerate(g["shards"]):
            rows = oracle.shard_rows(x, s, nshards)
            rs = oracle.cv_sorted(x, y, h, kid, rows=rows)
            part = np.asarray(part)
            assert cv_rel_err(part[:m], rs.S) <= TOL, (c, G, s)
            assert np.array_equal(part[m:2 * m].astype(np.int64), rs.neff), (c, G, s)
            assert part[2 * m] == 0 and part[2 * m + 1] == 0


def test_gxg_auto_selected_at_400k_rows():
    """n = 450,000 (>= kGxgRows): KR_ALGO_SWEEP auto-selects gxg for the whole
    search.  Its CV curve, n_eff and best against the window-prefix path on
    the same input (the oracle cannot run 450,000 full rows in a test; gxg's
    oracle parity is the forced test above)."""
    from paper_conf_ipps_rohlfsz17_b200 import krcv

    rng = np.random.default_rng(5)
    n, m = 450_000, 12
    x = rng.uniform(0, 1, n)
    y = 0.5 * x + 10 * x * x + rng.uniform(0, 0.5, n)
    h = np.geomspace(2e-5, 1.0, m)
    cv_s, ne_s, b_s = krcv.kr_cv_grid(x, y, h, 1, with_neff=True, algo="sweep")
    cv_p, ne_p, b_p = krcv.kr_cv_grid(x, y, h, 1, with_neff=True, algo="prefix")
    assert cv_rel_err(cv_s, cv_p) <= TOL
    assert np.array_equal(ne_s, ne_p)
    assert b_s == b_p
