"""Shared test helpers (no method arithmetic)."""
from __future__ import annotations

import numpy as np


def cv_rel_err(got, ref, abs_floor: float = 0.0) -> float:
    """max_b |got-ref| / max(|ref_b|, 1e-12 * max|ref|)  (SURVEY.md §8(c) parity rule).

    ``abs_floor`` raises the floor for inputs whose exact CV is 0 at every
    bandwidth (constant y, P6): there max|ref| is itself rounding noise (the
    oracle's long-double quotient 3w/w need not round to 3), so the relative
    floor would compare noise with noise; callers pass a value tied to the
    scale of y^2, far below any real discrepancy."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    floor = 1e-12 * float(np.max(np.abs(ref))) if ref.size else 0.0
    floor = max(floor, abs_floor, 1e-300)
    den = np.maximum(np.abs(ref), floor)
    return float(np.max(np.abs(got - ref) / den)) if ref.size else 0.0


def best_ok(best_got: int, cv_ref, tol: float = 1e-6, abs_tol: float = 0.0) -> bool:
    """north_star arg-min rule: identical index unless the reference's two best
    values lie within tol (then any index within tol of the minimum is fine);
    ``abs_tol`` as cv_rel_err's ``abs_floor`` (values below it are ties at 0)."""
    cv_ref = np.asarray(cv_ref, np.float64)
    finite = np.where(np.isnan(cv_ref), np.inf, cv_ref)
    b = int(np.argmin(finite))
    if best_got == b:
        return True
    return bool(finite[best_got] <= finite[b] * (1 + tol) + max(abs_tol, 1e-300))
