"""Window-prefix checker (pin P10, SURVEY.md §8(c) "Independent checkers").

TEST INFRASTRUCTURE ONLY.

An algorithm independent of both C evaluators: sort x once (stable); for each
bandwidth, the window of every row is a contiguous index range of the sorted
array, found with ``searchsorted`` and then corrected with the exact binary64
membership predicate of reading Q1 (d = x_q - x_p or x_p - x_q, '<' or '<='),
so membership equals the oracle's.  Window sums come from prefix sums of
*centred* moments in numpy long double; the LOO estimate is then assembled from
the Epanechnikov / triangular / uniform decompositions (Eq.(2)-(3), P@11694,
P@11971, footnote 1 P@18521), rows with an empty window are M = 0 (Q6, Q7).

Cost O(m n log n): usable at n = 1e5 .. 1e6.  Tolerance-only (the centred
prefix differences round differently from a direct sum): ~1e-12 on the
configs; no cancellation guard, so adversarial edge inputs are out of scope.
"""
from __future__ import annotations

import numpy as np

UNIFORM, EPANECHNIKOV, TRIANGULAR = 0, 1, 2
LD = np.longdouble


def _inside(d, h, kernel):
    return (d <= h) if kernel == UNIFORM else (d < h)


def _bounds(xs, h, kernel):
    """R[p] = first q > p outside the right window; L[p] = last q < p outside
    the left window (so the window is the open range (L, R) minus p)."""
    n = xs.shape[0]
    p = np.arange(n)
    side = "right" if kernel == UNIFORM else "left"
    R = np.searchsorted(xs, xs + h, side=side)
    R = np.maximum(R, p + 1)
    while True:  # fix-up with the exact predicate
        up = (R < n) & _inside(xs[np.minimum(R, n - 1)] - xs, h, kernel)
        dn = (R - 1 > p) & ~_inside(xs[np.maximum(R - 1, 0)] - xs, h, kernel)
        if not (up.any() or dn.any()):
            break
        R = R + up.astype(np.int64) - dn.astype(np.int64)
    side = "left" if kernel == UNIFORM else "right"
    L = np.searchsorted(xs, xs - h, side=side) - 1
    L = np.minimum(L, p - 1)
    while True:
        dn = (L >= 0) & _inside(xs - xs[np.maximum(L, 0)], h, kernel)
        up = (L + 1 < p) & ~_inside(xs - xs[np.minimum(L + 1, n - 1)], h, kernel)
        if not (up.any() or dn.any()):
            break
        L = L - dn.astype(np.int64) + up.astype(np.int64)
    return L, R


def cv_window(x, y, h, kernel: int, rows_sorted_pos=None):
    """Return dict(cv, S, neff, best).  rows_sorted_pos: optional slice of
    sorted positions (shard) to restrict the rows summed."""
    x = np.asarray(x, np.float64)
    y = np.asarray(y, np.float64)
    h = np.asarray(h, np.float64)
    n, m = x.shape[0], h.shape[0]
    order = np.argsort(x, kind="stable")
    xs, ys = x[order], y[order]
    c0 = xs[n // 2]
    t = xs.astype(LD) - LD(c0)
    yl = ys.astype(LD)

    def pre(v):
        out = np.zeros(n + 1, dtype=LD)
        np.cumsum(v, out=out[1:])
        return out

    P1, P2 = pre(t), pre(t * t)
    Py, Pyt, Pyt2 = pre(yl), pre(yl * t), pre(yl * t * t)
    sel = np.arange(n) if rows_sorted_pos is None else np.asarray(rows_sorted_pos)
    S = np.zeros(m, dtype=LD)
    neff = np.zeros(m, dtype=np.int64)
    p = np.arange(n)
    for b in range(m):
        L, R = _bounds(xs, h[b], kernel)
        L, R, pp = L[sel], R[sel], p[sel]
        tp, yp = t[sel], yl[sel]
        # right window [pp+1, R), left window [L+1, pp)
        def rng(P, a, bb):
            return P[bb] - P[a]
        cR = (R - pp - 1).astype(LD)
        cL = (pp - L - 1).astype(LD)
        c = cR + cL
        sy = rng(Py, pp + 1, R) + rng(Py, L + 1, pp)
        H = LD(h[b])
        if kernel == UNIFORM:
            num, den = sy, c
        elif kernel == EPANECHNIKOV:
            s1 = rng(P1, pp + 1, R) + rng(P1, L + 1, pp)
            s2 = rng(P2, pp + 1, R) + rng(P2, L + 1, pp)
            syt = rng(Pyt, pp + 1, R) + rng(Pyt, L + 1, pp)
            syt2 = rng(Pyt2, pp + 1, R) + rng(Pyt2, L + 1, pp)
            sd2 = s2 - 2 * tp * s1 + tp * tp * c
            syd2 = syt2 - 2 * tp * syt + tp * tp * sy
            num, den = H * H * sy - syd2, H * H * c - sd2
        else:
            s1R = rng(P1, pp + 1, R) - tp * cR
            s1L = tp * cL - rng(P1, L + 1, pp)
            sytR = rng(Pyt, pp + 1, R) - tp * rng(Py, pp + 1, R)
            sytL = tp * rng(Py, L + 1, pp) - rng(Pyt, L + 1, pp)
            num = H * sy - (sytR + sytL)
            den = H * c - (s1R + s1L)
        ok = c > 0
        g = np.where(ok, num / np.where(ok, den, LD(1)), LD(0))
        e = np.where(ok, yp - g, LD(0))
        S[b] = np.sum(e * e)
        neff[b] = int(np.count_nonzero(ok))
    cv = (S / LD(n)).astype(np.float64)
    finite = np.where(np.isnan(cv), np.inf, cv)
    best = int(np.argmin(finite))
    return {"cv": cv, "S": S.astype(np.float64), "neff": neff, "best": best}
