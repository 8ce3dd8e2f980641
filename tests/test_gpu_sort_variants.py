"""GPU: every a2 sort implementation gives the same total order.

The chunked rank sort (the default for n <= 131,072), the 32-bit quantised-key radix sort with its exact fix-up (KRCV_SORT=q32) and
CUB's 64-bit onesweep (KRCV_SORT=cub64) must all order the records by
(x, original index).  Identical sorted arrays make every later stage
bit-identical, so the CV curves, n_eff and best are compared bit for bit.
The library reads the selection once per process: one subprocess per
variant.  Sizes cover one chunk, a ragged last chunk, both chunk sizes (512
up to n = 40,000, 1,024 above), the rank sort's limit and the q32 default
above it; inputs include heavy duplicates, all-equal x, two values and a
heavy tail.
"""
from __future__ import annotations

import numpy as np
import pytest

from tests.test_gpu_window_variants import _run

pytestmark = pytest.mark.gpu

VARIANTS = {"rank": {"KRCV_SORT": "rank"}, "q32": {"KRCV_SORT": "q32"}, "cub64": {"KRCV_SORT": "cub64"}}


@pytest.fixture(scope="module")
def sort_cases(tmp_path_factory):
    import workloads

    rng = np.random.default_rng(23)
    cases = {}
    for cfg, n in (("C1", 1000), ("C2", 513), ("C2", 4097), ("C2", 20000), ("C2", 40001), ("C5", 5000),
                   ("C2", 131072)):
        x, y, h, k = workloads.make(cfg, seed=5, n=n)
        cases[f"{cfg}_{n}"] = (x, y, h[:: max(1, h.shape[0] // 24)].copy(), workloads.KERNEL_NAMES[k])
    x = np.floor(rng.uniform(0, 1, 9000) * 7) / 7
    cases["dups"] = (x, rng.normal(0, 1, 9000), np.linspace(0.05, 1.0, 12), "epanechnikov")
    cases["const"] = (np.full(2000, 0.25), rng.normal(0, 1, 2000), np.array([0.1, 1.0]), "epanechnikov")
    cases["two"] = (np.repeat([-1.0, 2.0], 1500)[rng.permutation(3000)], rng.normal(0, 1, 3000),
                    np.array([1.0, 3.0, 4.0]), "uniform")
    x = rng.lognormal(0, 2, 30000)
    cases["tail"] = (x, np.sin(x), np.geomspace(1e-3, x.max(), 16), "epanechnikov")
    path = str(tmp_path_factory.mktemp("sorts") / "cases.npz")
    arrs = {}
    for c, (x, y, h, k) in cases.items():
        arrs[c + "_x"], arrs[c + "_y"], arrs[c + "_h"], arrs[c + "_k"] = x, y, h, np.array(k)
    np.savez(path, **arrs)
    return path, cases


@pytest.fixture(scope="module")
def rank_result(sort_cases):
    return _run(VARIANTS["rank"], sort_cases[0])


@pytest.mark.parametrize("variant", ["q32", "cub64"])
def test_sorts_give_identical_results(sort_cases, rank_result, variant):
    path, cases = sort_cases
    b = _run(VARIANTS[variant], path)
    for c in cases:
        assert rank_result[c]["cv"] == b[c]["cv"], (c, variant)
        assert rank_result[c]["neff"] == b[c]["neff"], (c, variant)
        assert rank_result[c]["best"] == b[c]["best"], (c, variant)


def test_rank_sort_matches_oracle(sort_cases, rank_result):
    import oracle
    from tests.helpers import best_ok, cv_rel_err

    path, cases = sort_cases
    kid = {"uniform": 0, "epanechnikov": 1, "triangular": 2}
    for c in ("C2_4097", "dups", "const", "two", "C1_1000"):
        x, y, h, k = cases[c]
        ref = oracle.cv_sorted(x, y, h, kid[k])
        got = np.array(rank_result[c]["cv"], np.uint64).view(np.float64)
        assert cv_rel_err(got, ref.cv) <= 1e-10, c
        assert np.array_equal(np.asarray(rank_result[c]["neff"]), ref.neff), c
        assert best_ok(rank_result[c]["best"], ref.cv), c
