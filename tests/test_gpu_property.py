"""Property-based GPU parity (hypothesis): random small inputs -- duplicate
x, points exactly at a bandwidth, wide dynamic range, tiny and huge h,
unsorted grids with repeats -- through every algorithm of the C-ABI against
the oracle.  Integer results (n_eff) must match exactly; CV to 1e-9
(relative, with the floor of tests/helpers.cv_rel_err); best by the tie rule.
"""
from __future__ import annotations

import numpy as np
import pytest
from hypothesis import HealthCheck, example, given, settings
from hypothesis import strategies as st

import oracle
from paper_conf_ipps_rohlfsz17_b200 import krcv
from tests.helpers import best_ok, cv_rel_err

pytestmark = pytest.mark.gpu

TOL = 1e-9


@st.composite
def problems(draw):
    n = draw(st.integers(2, 48))
    scale = draw(st.sampled_from([1.0, 1e-6, 1e4]))
    if draw(st.booleans()):  # dyadic grid of positions: exact distances, many ties
        xi = draw(st.lists(st.integers(0, 24), min_size=n, max_size=n))
        x = np.array(xi, np.float64) / 8.0 * scale
    else:
        # 12 decimals: distinct x differ by >= 1e-12 * scale, so d^2 never
        # underflows binary64 (the long-double oracle would not underflow)
        x = np.array(draw(st.lists(st.floats(-1.0, 1.0, allow_nan=False, width=64).map(lambda v: round(v, 12)),
                                   min_size=n, max_size=n)))
        x = x * scale
    y = np.array(draw(st.lists(st.floats(-4.0, 4.0, allow_nan=False, width=64), min_size=n, max_size=n)))
    m = draw(st.integers(1, 8))
    d = np.abs(x[:, None] - x[None, :])
    pos = d[d > 0]
    cands = list(pos[:16]) if pos.size else []
    hs = []
    for _ in range(m):
        if cands and draw(st.booleans()):
            hs.append(float(cands[draw(st.integers(0, len(cands) - 1))]))  # exactly at a pair distance
        else:
            hs.append(scale * draw(st.floats(1e-3, 4.0, allow_nan=False)))
    h = np.sort(np.array(hs, np.float64))
    return x, y, h


# derandomize: the same examples on every run (the round-end GPU run must be
# reproducible); the example set was widened instead (max_examples)
SETTINGS = settings(max_examples=60, deadline=None, derandomize=True, database=None,
                    suppress_health_check=[HealthCheck.too_slow])


def zero_floor(y) -> float:
    """Floor for exact-zero CV (constant y, P6; helpers.cv_rel_err): fp64 noise
    there is ~1e-32 max y^2 (measured 1.4e-32 y^2, hist/triangular, n = 2), and
    TOL times the floor must exceed it; 1e-20 max y^2 allows 1e-29 y^2 at
    TOL = 1e-9, while one misplaced window member changes CV by O(y^2 / n)."""
    return 1e-20 * float(np.max(np.asarray(y) ** 2))


@pytest.mark.parametrize("algo", ["sweep", "prefix", "hist"])
@pytest.mark.parametrize("k", [0, 1, 2])
@SETTINGS
@given(p=problems())
# found by random runs: constant y, exact CV 0, the oracle's triangular
# quotient leaves 4.7e-38, the GPU's 4.9e-32 (zero_floor)
@example(p=(np.array([0.0, 1.625]), np.array([3.0, 3.0]), np.array([3.0])))
@example(p=(np.array([0.0, 0.0]), np.array([1.875, 1.875]), np.array([2.18257963])))
def test_property_nw(algo, k, p):
    x, y, h = p
    cv, neff, best = krcv.kr_cv_grid(x, y, h, k, with_neff=True, algo=algo)
    ref = oracle.cv_direct(x, y, h, k)
    assert np.array_equal(neff, ref.neff)
    assert cv_rel_err(cv, ref.cv, zero_floor(y)) <= TOL
    assert best_ok(best, ref.cv, 1e-9, zero_floor(y))


@pytest.mark.parametrize("k", [0, 1, 2])
@SETTINGS
@given(p=problems())
def test_property_local_linear(k, p):
    x, y, h = p
    cv, neff, best = krcv.kr_ll_cv_grid(x, y, h, k, with_neff=True)
    ref = oracle.ll_cv(x, y, h, k)
    assert np.array_equal(neff, ref.neff)
    assert cv_rel_err(cv, ref.cv, zero_floor(y)) <= 1e-7  # ill-conditioned 2-point fits amplify rounding
    assert best_ok(best, ref.cv, 1e-7, zero_floor(y))


@SETTINGS
@given(p=problems())
def test_property_gaussian(p):
    x, y, h = p
    cv, neff, best = krcv.kr_cv_grid(x, y, h, 3, with_neff=True)
    ref = oracle.cv_direct(x, y, h, 3)
    assert np.array_equal(neff, ref.neff)
    assert cv_rel_err(cv, ref.cv, zero_floor(y)) <= TOL
