"""CPU oracle for the LOO-CV bandwidth grid search (Rohlfs & Zahran 2017).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with the CUDA path; the only module both sides
import is ``workloads`` (seeded input recipes, no method arithmetic).

Contents
--------
* ``cv_direct``   -- C, the plain definition Eq.(1)-(3) (PAPER.md P@11484-12036),
                     O(n^2 m), long double (or double for pin P9).
* ``cv_sorted``   -- C, the paper's Program 3: per-row sort + ascending sweep
                     (P@13614-14984, P@20401-22459), long double.
* ``exact.cv_exact``        -- Python ``fractions`` brute force of Eq.(1)-(3).
* ``window.cv_window``      -- numpy long-double window-prefix checker (pin P10).
* ``ll_cv``       -- C, local-linear LOO CV by its plain definition
                     (weighted least-squares intercept, centred two-pass form;
                     PAPER.md P@15728, reading Q25), O(n^2 m), long double.
* ``exact.ll_cv_exact``     -- Python ``fractions`` brute force of the
                               local-linear normal equations.
* ``nw_jackknife`` / ``kde_jackknife`` -- C, leave-one-out (delete-one
                     jackknife) confidence intervals at a bandwidth (PAPER.md
                     P@10560, reading Q26), plain definitions, long double;
                     ``cv_ci`` / ``kde_ci`` run them at the CV / LSCV optimum.
* ``exact.nw_jackknife_exact`` / ``exact.kde_jackknife_exact`` -- Python
                     ``fractions``: the jackknife by explicit deletion.
* ``sorted_rows``           -- the x-sorted row order (stable by (x, index))
                               that defines shards.

Parity status: every function here is pinned by tests/test_oracle_pins.py
(see DESIGN.md "Oracle pins").  None is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_BUILD = os.path.join(_HERE, "build")

UNIFORM, EPANECHNIKOV, TRIANGULAR, GAUSSIAN = 0, 1, 2, 3

_libs: dict[str, ctypes.CDLL] = {}


def build() -> None:
    """Compile the oracle shared libraries (gcc + OpenMP)."""
    subprocess.run(["make", "-s", "-C", _HERE], check=True)


def _lib(precision: str = "ld") -> ctypes.CDLL:
    if precision not in ("ld", "d"):
        raise ValueError(precision)
    if precision in _libs:
        return _libs[precision]
    path = os.path.join(_BUILD, f"liboracle_{precision}.so")
    if not os.path.exists(path):
        build()
    lib = ctypes.CDLL(path)
    P = ctypes.c_void_p
    i64, i32 = ctypes.c_int64, ctypes.c_int32
    lib.kro_cv_direct.argtypes = [P, P, i64, P, i32, i32, P, i64, P, P, P, P, P, P, P]
    lib.kro_cv_direct.restype = ctypes.c_int
    lib.kro_cv_sorted.argtypes = [P, P, i64, P, i32, i32, P, i64, P, P, P, P]
    lib.kro_cv_sorted.restype = ctypes.c_int
    lib.kro_default_grid.argtypes = [P, i64, i32, P]
    lib.kro_default_grid.restype = ctypes.c_int
    lib.kro_finalize.argtypes = [P, i64, i32, P, P]
    lib.kro_finalize.restype = ctypes.c_int
    lib.kro_kde_lscv.argtypes = [P, i64, P, i32, i32, P, i64, P, P, P, P]
    lib.kro_kde_lscv.restype = ctypes.c_int
    lib.kro_ll_cv.argtypes = [P, P, i64, P, i32, i32, P, i64, P, P, P, P]
    lib.kro_ll_cv.restype = ctypes.c_int
    lib.kro_nw_jackknife.argtypes = [P, P, i64, ctypes.c_double, i32, P, P, P]
    lib.kro_nw_jackknife.restype = ctypes.c_int
    lib.kro_kde_jackknife.argtypes = [P, i64, ctypes.c_double, i32, P, P]
    lib.kro_kde_jackknife.restype = ctypes.c_int
    lib.kro_real_bits.restype = ctypes.c_int
    lib.kro_num_threads.restype = ctypes.c_int
    _libs[precision] = lib
    return lib


class OracleError(RuntimeError):
    def __init__(self, status: int):
        super().__init__(f"oracle status {status}")
        self.status = status


def _ptr(a):
    return None if a is None else a.ctypes.data


def _prep(x, y, h):
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.ascontiguousarray(y, dtype=np.float64)
    h = np.ascontiguousarray(h, dtype=np.float64)
    return x, y, h


class Result(dict):
    """dict with keys cv, best, S, neff (and aux sums for cv_direct)."""
    __getattr__ = dict.__getitem__


def cv_direct(x, y, h, kernel: int, rows=None, precision: str = "ld", aux: bool = False) -> Result:
    """Plain definition, Eq.(1)-(3).  rows: optional original-index row list."""
    x, y, h = _prep(x, y, h)
    n, m = x.shape[0], h.shape[0]
    r = None if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    S = np.zeros(m); ne = np.zeros(m, np.int64); cv = np.zeros(m)
    best = ctypes.c_int32(-1)
    cs = np.zeros(m, np.int64) if aux else None
    sy = np.zeros(m) if aux else None
    s2 = np.zeros(m) if aux else None
    st = _lib(precision).kro_cv_direct(
        _ptr(x), _ptr(y), n, _ptr(h), m, int(kernel), _ptr(r), 0 if r is None else r.shape[0],
        _ptr(S), _ptr(ne), _ptr(cs), _ptr(sy), _ptr(s2), _ptr(cv), ctypes.byref(best))
    if st:
        raise OracleError(st)
    out = Result(cv=cv, best=int(best.value), S=S, neff=ne)
    if aux:
        out.update(csum=cs, sysum=sy, sd2sum=s2)
    return out


def cv_sorted(x, y, h, kernel: int, rows=None, precision: str = "ld") -> Result:
    """The paper's Program-3 algorithm: per-row sort + ascending sweep."""
    x, y, h = _prep(x, y, h)
    n, m = x.shape[0], h.shape[0]
    r = None if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    S = np.zeros(m); ne = np.zeros(m, np.int64); cv = np.zeros(m)
    best = ctypes.c_int32(-1)
    st = _lib(precision).kro_cv_sorted(
        _ptr(x), _ptr(y), n, _ptr(h), m, int(kernel), _ptr(r), 0 if r is None else r.shape[0],
        _ptr(S), _ptr(ne), _ptr(cv), ctypes.byref(best))
    if st:
        raise OracleError(st)
    return Result(cv=cv, best=int(best.value), S=S, neff=ne)


def default_grid(x, m: int) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float64)
    h = np.zeros(m)
    st = _lib().kro_default_grid(_ptr(x), x.shape[0], int(m), _ptr(h))
    if st:
        raise OracleError(st)
    return h


def finalize(S, n: int):
    """CV = S/n and the Q11 arg-min, for summed shard partials."""
    S = np.ascontiguousarray(S, dtype=np.float64)
    m = S.shape[0]
    cv = np.zeros(m); best = ctypes.c_int32(-1)
    st = _lib().kro_finalize(_ptr(S), int(n), m, _ptr(cv), ctypes.byref(best))
    if st:
        raise OracleError(st)
    return cv, int(best.value)


def sorted_rows(x) -> np.ndarray:
    """Row order of the x-sorted data, ties by original index (stable)."""
    return np.argsort(np.asarray(x, dtype=np.float64), kind="stable").astype(np.int64)


def shard_rows(x, shard: int, nshards: int) -> np.ndarray:
    """Original indices of the rows of shard r/P: sorted positions
    [floor(r n / P), floor((r+1) n / P))."""
    order = sorted_rows(x)
    n = order.shape[0]
    lo, hi = (shard * n) // nshards, ((shard + 1) * n) // nshards
    return order[lo:hi]


def num_threads() -> int:
    return int(_lib().kro_num_threads())


def real_bits(precision: str = "ld") -> int:
    return int(_lib(precision).kro_real_bits())


def refine_grid(h, best: int, m_fine: int) -> np.ndarray:
    """Level l+1 grid of the coarse-to-fine search (§IV.A P@20112-20269:
    "run the optimization code multiple times with progressively smaller
    ranges of possible bandwidths"; the range rule is reading Q22, DESIGN.md
    §2): m_fine evenly spaced points on [lo, hi], lo = h[b-1] (h[b]/2 if b is
    the first index), hi = h[b+1] (2 h[b] if b is the last), both ends
    included: h_j = lo + (hi - lo) * (j / (m_fine - 1)), the last point = hi."""
    h = [float(v) for v in h]
    m = len(h)
    lo = h[best - 1] if best > 0 else h[best] / 2.0
    hi = h[best + 1] if best < m - 1 else 2.0 * h[best]
    out = []
    for j in range(m_fine):
        t = float(j) / float(m_fine - 1)
        out.append(lo + (hi - lo) * t)
    out[-1] = hi
    return np.array(out, dtype=np.float64)


def cv_refine(x, y, h, kernel: int, levels: int, m_fine: int, evaluate=None):
    """Coarse-to-fine search: level 0 on h, each next level on refine_grid
    around the previous level's best index.  `evaluate(x, y, h, kernel)`
    returns an object with .cv and .best (default: cv_sorted).  Returns
    (h_best[levels], cv_best[levels], grids)."""
    evaluate = evaluate or (lambda a, b, g, k: cv_sorted(a, b, g, k))
    grid = np.asarray(h, dtype=np.float64)
    hb, cb, grids = [], [], []
    for level in range(levels):
        grids.append(grid)
        r = evaluate(x, y, grid, kernel)
        hb.append(float(grid[r.best]))
        cb.append(float(r.cv[r.best]))
        if level + 1 < levels:
            grid = refine_grid(grid, r.best, m_fine)
    return np.array(hb), np.array(cb), grids


def kde_lscv(x, h, kernel: int, rows=None, precision: str = "ld") -> Result:
    """KDE least-squares cross-validation by the plain definition (PAPER.md
    P@10382-10640; reading Q24): lscv[m] (full rows only), the per-bandwidth
    row sums A (sum of Kbar over pairs, Kbar = K*K) and B (sum of K over
    pairs) over `rows` (default: all), best index."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    h = np.ascontiguousarray(h, dtype=np.float64)
    n, m = x.shape[0], h.shape[0]
    r = None if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    A = np.empty(m)
    B = np.empty(m)
    lscv = np.full(m, np.nan)
    best = ctypes.c_int32(-1)
    st = _lib(precision).kro_kde_lscv(x.ctypes.data, n, h.ctypes.data, m, int(kernel), _ptr(r),
                                      0 if r is None else r.shape[0], A.ctypes.data, B.ctypes.data,
                                      lscv.ctypes.data, ctypes.byref(best))
    if st:
        raise OracleError(st)
    return Result(lscv=lscv, A=A, B=B, best=int(best.value))


def ll_cv(x, y, h, kernel: int, rows=None, precision: str = "ld") -> Result:
    """Local-linear LOO CV by the plain definition (reading Q25): for every
    bandwidth and row, the intercept of the kernel-weighted least-squares line
    through the in-window neighbours (row excluded); M_i = [>= 2 distinct x in
    the window].  Returns cv, best, S (sum of M e^2 over `rows`), neff."""
    x, y, h = _prep(x, y, h)
    n, m = x.shape[0], h.shape[0]
    r = None if rows is None else np.ascontiguousarray(rows, dtype=np.int64)
    S = np.zeros(m); ne = np.zeros(m, np.int64); cv = np.zeros(m)
    best = ctypes.c_int32(-1)
    st = _lib(precision).kro_ll_cv(
        _ptr(x), _ptr(y), n, _ptr(h), m, int(kernel), _ptr(r), 0 if r is None else r.shape[0],
        _ptr(S), _ptr(ne), _ptr(cv), ctypes.byref(best))
    if st:
        raise OracleError(st)
    return Result(cv=cv, best=int(best.value), S=S, neff=ne)


def nw_jackknife(x, y, h: float, kernel: int, precision: str = "ld") -> Result:
    """Delete-one jackknife interval pieces for the Nadaraya-Watson estimate at
    every observation at bandwidth h (reading Q26): est[n] (full-sample
    estimate, the point itself included), se[n] (NaN where the window holds
    only the point), nwin[n] (window sizes)."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.ascontiguousarray(y, dtype=np.float64)
    n = x.shape[0]
    est, se, nw = np.empty(n), np.empty(n), np.empty(n, np.int64)
    st = _lib(precision).kro_nw_jackknife(x.ctypes.data, y.ctypes.data, n, float(h), int(kernel),
                                          est.ctypes.data, se.ctypes.data, nw.ctypes.data)
    if st:
        raise OracleError(st)
    return Result(est=est, se=se, nwin=nw)


def kde_jackknife(x, h: float, kernel: int, precision: str = "ld") -> Result:
    """Delete-one jackknife interval pieces for the kernel density estimate at
    every observation at bandwidth h (reading Q26): est[n] = f_h(x_i), se[n]."""
    x = np.ascontiguousarray(x, dtype=np.float64)
    n = x.shape[0]
    est, se = np.empty(n), np.empty(n)
    st = _lib(precision).kro_kde_jackknife(x.ctypes.data, n, float(h), int(kernel), est.ctypes.data,
                                           se.ctypes.data)
    if st:
        raise OracleError(st)
    return Result(est=est, se=se)


def cv_ci(x, y, h, kernel: int) -> Result:
    """The CV-optimal bandwidth (Program 3, cv_sorted) and the jackknife
    interval pieces there (reading Q26): best, h_best, est, se, nwin."""
    r = cv_sorted(x, y, h, kernel)
    hb = float(np.asarray(h, dtype=np.float64)[r.best])
    j = nw_jackknife(x, y, hb, kernel)
    return Result(best=r.best, h_best=hb, est=j.est, se=j.se, nwin=j.nwin)


def kde_ci(x, h, kernel: int) -> Result:
    """The LSCV-optimal bandwidth (kde_lscv) and the jackknife interval pieces
    of the density estimate there (reading Q26): best, h_best, est, se."""
    r = kde_lscv(x, h, kernel)
    hb = float(np.asarray(h, dtype=np.float64)[r.best])
    j = kde_jackknife(x, hb, kernel)
    return Result(best=r.best, h_best=hb, est=j.est, se=j.se)
