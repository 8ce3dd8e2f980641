"""Thin ctypes binding of ``libkrcv.so`` (include/krcv.h).

Argument marshalling only: every step of the hot path runs in the sm_100a
kernels of ``csrc/krcv_device.cu``.  There is no CPU fallback: if the shared
library is missing the import fails loudly (build it with
``python -c "import __graft_entry__ as g; g.build()"``).

The functions keep the C names (``kr_cv_grid``, ``kr_cv_shard_async``,
``kr_finalize``, ``kr_finalize_async``, ``kr_default_grid``,
``kr_workspace_bytes``, ``kr_validate_grid``, ``kr_strerror``).
Host-pointer calls take numpy arrays; device-pointer calls take
``torch.Tensor`` objects on a CUDA device (PyTorch provides device memory and
streams only).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# KRCV_LIB selects another in-tree build variant of the same library (A/B
# measurements of compile-time options, tools/); default libkrcv.so
LIB_PATH = os.path.join(_HERE, os.environ.get("KRCV_LIB", "libkrcv.so"))

UNIFORM, EPANECHNIKOV, TRIANGULAR, GAUSSIAN = 0, 1, 2, 3
KERNELS = {"uniform": UNIFORM, "epanechnikov": EPANECHNIKOV, "triangular": TRIANGULAR, "gaussian": GAUSSIAN}

ALGO_AUTO, ALGO_SWEEP, ALGO_PREFIX, ALGO_DENSE, ALGO_HIST = 0, 1, 2, 3, 4
ALGOS = {"auto": ALGO_AUTO, "sweep": ALGO_SWEEP, "prefix": ALGO_PREFIX, "dense": ALGO_DENSE, "hist": ALGO_HIST}

KR_OK, KR_EARG, KR_EKERNEL, KR_EGRID, KR_ENONFINITE, KR_EDEGENERATE, KR_ENOMEM, KR_ECUDA = range(8)
KR_MAX_M = 65536

# Every symbol include/krcv.h declares (checked by tests/test_abi.py).
EXPORTS = (
    "kr_cv_grid", "kr_cv_grid_ex", "kr_cv_grid_algo", "kr_cv_refine", "kr_validate_grid", "kr_workspace_bytes",
    "kr_cv_shard_async", "kr_cv_shard_algo_async", "kr_cv_rows_async", "kr_cv_grid_async", "kr_finalize", "kr_finalize_async", "kr_default_grid",
    "kr_strerror", "kr_last_cuda_error", "kr_version", "kr_release",
    "kr_profile_enable", "kr_profile_read", "kr_launch_count", "kr_last_algo",
    "kr_kde_lscv", "kr_kde_lscv_async", "kr_kde_shard_async", "kr_kde_finalize",
    "kr_ll_cv_grid", "kr_ll_cv_grid_async", "kr_ll_shard_async",
    "kr_cv_ci", "kr_kde_ci", "kr_cv_ci_async", "kr_kde_ci_async",
    "kr_workspace_bytes_algo", "kr_kde_workspace_bytes",
)


def partial_len(m: int) -> int:
    return 2 * int(m) + 2


class KrcvError(RuntimeError):
    def __init__(self, status: int, where: str = ""):
        msg = _lib().kr_strerror(status).decode()
        if status == KR_ECUDA:
            msg += f": {_lib().kr_last_cuda_error().decode()}"
        super().__init__(f"{where}: {msg} (status {status})" if where else msg)
        self.status = status


_LIB = None


def _lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise ImportError(
            f"libkrcv.so not found at {LIB_PATH}; build it with __graft_entry__.build() "
            "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    P, i64, i32, sz = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_size_t
    lib.kr_cv_grid.argtypes = [P, P, i64, P, i32, i32, P, P]
    lib.kr_cv_grid_ex.argtypes = [P, P, i64, P, i32, i32, P, P, P]
    lib.kr_cv_grid_algo.argtypes = [P, P, i64, P, i32, i32, i32, P, P, P]
    lib.kr_cv_refine.argtypes = [P, P, i64, P, i32, i32, i32, i32, i32, P, P]
    lib.kr_validate_grid.argtypes = [P, i32]
    lib.kr_workspace_bytes.argtypes = [i64, i32]
    lib.kr_workspace_bytes.restype = sz
    lib.kr_workspace_bytes_algo.argtypes = [i64, i32, i32, i32]
    lib.kr_workspace_bytes_algo.restype = sz
    lib.kr_kde_workspace_bytes.argtypes = [i64, i32]
    lib.kr_kde_workspace_bytes.restype = sz
    lib.kr_cv_shard_async.argtypes = [P, P, i64, P, i32, i32, i32, i32, P, P, sz, P]
    lib.kr_cv_shard_algo_async.argtypes = [P, P, i64, P, i32, i32, i32, i32, i32, P, P, sz, P]
    lib.kr_cv_rows_async.argtypes = [P, P, i64, P, i32, i32, i32, i64, i64, P, P, sz, P]
    lib.kr_cv_grid_async.argtypes = [P, P, i64, P, i32, i32, i32, P, P, P, P, sz, P]
    lib.kr_finalize.argtypes = [P, i64, i32, P, P, P]
    lib.kr_finalize_async.argtypes = [P, i64, i32, P, P, P, P, P]
    lib.kr_default_grid.argtypes = [P, i64, i32, P]
    for f in ("kr_cv_grid", "kr_cv_grid_ex", "kr_cv_grid_algo", "kr_cv_refine", "kr_validate_grid", "kr_cv_shard_async",
              "kr_cv_shard_algo_async", "kr_cv_rows_async", "kr_cv_grid_async",
              "kr_finalize", "kr_finalize_async", "kr_default_grid"):
        getattr(lib, f).restype = ctypes.c_int
    lib.kr_strerror.argtypes = [ctypes.c_int]
    lib.kr_strerror.restype = ctypes.c_char_p
    lib.kr_last_cuda_error.restype = ctypes.c_char_p
    lib.kr_version.restype = ctypes.c_char_p
    lib.kr_profile_enable.argtypes = [ctypes.c_int]
    lib.kr_profile_enable.restype = ctypes.c_int
    lib.kr_profile_read.argtypes = [P]
    lib.kr_profile_read.restype = ctypes.c_int
    lib.kr_launch_count.restype = ctypes.c_int64
    lib.kr_kde_lscv.argtypes = [P, i64, P, i32, i32, P, P]
    lib.kr_kde_lscv_async.argtypes = [P, i64, P, i32, i32, P, P, P, sz, P]
    lib.kr_kde_shard_async.argtypes = [P, i64, P, i32, i32, i32, i32, P, P, sz, P]
    lib.kr_kde_finalize.argtypes = [P, i64, P, i32, i32, P, P]
    for f in ("kr_kde_lscv", "kr_kde_lscv_async", "kr_kde_shard_async", "kr_kde_finalize"):
        getattr(lib, f).restype = ctypes.c_int
    lib.kr_ll_cv_grid.argtypes = [P, P, i64, P, i32, i32, P, P, P]
    lib.kr_ll_cv_grid_async.argtypes = [P, P, i64, P, i32, i32, P, P, P, P, sz, P]
    lib.kr_ll_shard_async.argtypes = [P, P, i64, P, i32, i32, i32, i32, P, P, sz, P]
    for f in ("kr_ll_cv_grid", "kr_ll_cv_grid_async", "kr_ll_shard_async"):
        getattr(lib, f).restype = ctypes.c_int
    lib.kr_cv_ci.argtypes = [P, P, i64, P, i32, i32, P, P, P, P]
    lib.kr_kde_ci.argtypes = [P, i64, P, i32, i32, P, P, P, P]
    lib.kr_cv_ci_async.argtypes = [P, P, i64, P, i32, i32, P, P, P, P, P, sz, P]
    lib.kr_kde_ci_async.argtypes = [P, i64, P, i32, i32, P, P, P, P, P, sz, P]
    for f in ("kr_cv_ci", "kr_kde_ci", "kr_cv_ci_async", "kr_kde_ci_async"):
        getattr(lib, f).restype = ctypes.c_int
    lib.kr_last_algo.restype = ctypes.c_int32
    _LIB = lib
    return lib


def _kernel_id(kernel) -> int:
    if isinstance(kernel, str):
        return KERNELS[kernel.lower()]
    return int(kernel)


def _algo_id(algo) -> int:
    if isinstance(algo, str):
        return ALGOS[algo.lower()]
    return int(algo)


def _host(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float64)


def _check(st: int, where: str) -> None:
    if st != KR_OK:
        raise KrcvError(st, where)


# ------------------------------------------------------------------ host API
def kr_cv_grid(x, y, h, kernel="epanechnikov", with_neff: bool = False, algo="auto"):
    """Whole grid search on the current CUDA device from host arrays.
    Returns (cv[m], best) or (cv, neff, best).  ``algo`` = "auto" | "sweep" |
    "prefix" (KR_ALGO_*); "auto" calls kr_cv_grid / kr_cv_grid_ex themselves."""
    x, y, h = _host(x), _host(y), _host(h)
    if x.shape != y.shape or x.ndim != 1:
        raise ValueError("x and y must be 1-D arrays of equal length")
    n, m = x.shape[0], h.shape[0]
    cv = np.empty(m, np.float64)
    best = ctypes.c_int32(-1)
    a = _algo_id(algo)
    if a != ALGO_AUTO:
        neff = np.empty(m, np.int64)
        st = _lib().kr_cv_grid_algo(x.ctypes.data, y.ctypes.data, n, h.ctypes.data, m, _kernel_id(kernel), a,
                                    cv.ctypes.data, neff.ctypes.data, ctypes.byref(best))
        _check(st, "kr_cv_grid_algo")
        return (cv, neff, int(best.value)) if with_neff else (cv, int(best.value))
    if with_neff:
        neff = np.empty(m, np.int64)
        st = _lib().kr_cv_grid_ex(x.ctypes.data, y.ctypes.data, n, h.ctypes.data, m, _kernel_id(kernel),
                                  cv.ctypes.data, neff.ctypes.data, ctypes.byref(best))
        _check(st, "kr_cv_grid_ex")
        return cv, neff, int(best.value)
    st = _lib().kr_cv_grid(x.ctypes.data, y.ctypes.data, n, h.ctypes.data, m, _kernel_id(kernel),
                           cv.ctypes.data, ctypes.byref(best))
    _check(st, "kr_cv_grid")
    return cv, int(best.value)


def kr_cv_refine(x, y, h, kernel="epanechnikov", levels: int = 3, m_fine: int = 65, algo="auto"):
    """Coarse-to-fine search (§IV.A P@20112): returns (h_best[levels], cv_best[levels])."""
    x, y, h = _host(x), _host(y), _host(h)
    if x.shape != y.shape or x.ndim != 1:
        raise ValueError("x and y must be 1-D arrays of equal length")
    hb = np.empty(int(levels), np.float64)
    cb = np.empty(int(levels), np.float64)
    st = _lib().kr_cv_refine(x.ctypes.data, y.ctypes.data, x.shape[0], h.ctypes.data, h.shape[0], _kernel_id(kernel),
                             _algo_id(algo), int(levels), int(m_fine), hb.ctypes.data, cb.ctypes.data)
    _check(st, "kr_cv_refine")
    return hb, cb


def kr_cv_grid_ptr(x_ptr: int, y_ptr: int, n: int, h_ptr: int, m: int, kernel: int,
                   cv_ptr: int, best_ref) -> int:
    """Raw-pointer form (used by bench.py's end-to-end leg with pinned buffers)."""
    return _lib().kr_cv_grid(x_ptr, y_ptr, n, h_ptr, m, kernel, cv_ptr, best_ref)


def kr_default_grid(x, m: int) -> np.ndarray:
    x = _host(x)
    h = np.empty(int(m), np.float64)
    _check(_lib().kr_default_grid(x.ctypes.data, x.shape[0], int(m), h.ctypes.data), "kr_default_grid")
    return h


def kr_validate_grid(h) -> int:
    h = _host(h)
    return int(_lib().kr_validate_grid(h.ctypes.data if h.size else None, h.shape[0]))


def kr_finalize(partial, n: int, m: int):
    """Host finalize of summed partials -> (cv, neff, best)."""
    p = _host(partial)
    if p.shape[0] != partial_len(m):
        raise ValueError("partial must have length 2m+2")
    cv = np.empty(m, np.float64)
    neff = np.empty(m, np.int64)
    best = ctypes.c_int32(-1)
    _check(_lib().kr_finalize(p.ctypes.data, int(n), int(m), cv.ctypes.data, neff.ctypes.data,
                              ctypes.byref(best)), "kr_finalize")
    return cv, neff, int(best.value)


def kr_strerror(status: int) -> str:
    return _lib().kr_strerror(int(status)).decode()


def kr_version() -> str:
    return _lib().kr_version().decode()


def kr_release() -> None:
    """Free the state the synchronous host entry points keep between calls."""
    _check(_lib().kr_release(), "kr_release")


def kr_workspace_bytes(n: int, m: int, kernel=None, algo=None, kde: bool = False) -> int:
    """Workspace bytes: for every entry point (default), for one algorithm
    (kernel and algo given: kr_workspace_bytes_algo) or for the KDE family."""
    if kde:
        return int(_lib().kr_kde_workspace_bytes(int(n), int(m)))
    if algo is not None:
        k = EPANECHNIKOV if kernel is None else _kernel_id(kernel)
        return int(_lib().kr_workspace_bytes_algo(int(n), int(m), k, _algo_id(algo)))
    return int(_lib().kr_workspace_bytes(int(n), int(m)))


# ---------------------------------------------------------------- device API
def _check_f64(name: str, t, numel=None) -> None:
    """Contiguous float64 CUDA tensor (of ``numel`` elements when given)."""
    import torch

    if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
        raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if numel is not None and t.numel() != numel:
        raise ValueError(f"{name} must have {numel} elements, got {t.numel()}")


def _check_best_status(t) -> None:
    """Exactly two contiguous int32 CUDA elements: (best, status)."""
    import torch

    if not (t.is_cuda and t.dtype == torch.int32 and t.is_contiguous() and t.numel() == 2):
        raise ValueError("best_status must be a contiguous int32 CUDA tensor of 2 elements")


def _check_neff(t, m: int) -> None:
    import torch

    if t is not None and not (t.is_cuda and t.dtype == torch.int64 and t.is_contiguous() and t.numel() == m):
        raise ValueError("neff must be None or a contiguous int64 CUDA tensor of m elements")


def kr_cv_rows_async(d_x, d_y, d_h, kernel, row_lo: int, row_hi: int, d_partial, d_ws, stream=None,
                     algo="auto") -> None:
    """Enqueue the device pipeline for rows [row_lo, row_hi) of the sorted
    order (cost-balanced sharding); tensors as kr_cv_shard_async."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    for t, name in ((d_x, "x"), (d_y, "y"), (d_h, "h"), (d_partial, "partial")):
        if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
            raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if d_partial.numel() != partial_len(m):
        raise ValueError("partial must have 2m+2 elements")
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    st = _lib().kr_cv_rows_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                 _algo_id(algo), int(row_lo), int(row_hi), d_partial.data_ptr(), d_ws.data_ptr(),
                                 d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream))
    _check(st, "kr_cv_rows_async")


def kr_cv_shard_async(d_x, d_y, d_h, kernel, shard: int, nshards: int, d_partial, d_ws, stream=None,
                      algo="auto") -> None:
    """Enqueue the sharded device pipeline.  All tensor arguments are CUDA
    torch tensors (float64 for x, y, h, partial; uint8 for the workspace).
    ``algo`` "auto" calls kr_cv_shard_async, otherwise kr_cv_shard_algo_async."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    for t, name in ((d_x, "x"), (d_y, "y"), (d_h, "h"), (d_partial, "partial")):
        if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
            raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if d_partial.numel() != partial_len(m):
        raise ValueError("partial must have 2m+2 elements")
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    a = _algo_id(algo)
    if a == ALGO_AUTO:
        st = _lib().kr_cv_shard_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                      int(shard), int(nshards), d_partial.data_ptr(), d_ws.data_ptr(),
                                      d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream))
        _check(st, "kr_cv_shard_async")
        return
    st = _lib().kr_cv_shard_algo_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                       a, int(shard), int(nshards), d_partial.data_ptr(), d_ws.data_ptr(),
                                       d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream))
    _check(st, "kr_cv_shard_algo_async")


def kr_cv_grid_async(d_x, d_y, d_h, kernel, d_cv, d_neff, d_best_status, d_ws, stream=None, algo="auto") -> None:
    """Enqueue the whole single-GPU search (fused finalize): d_cv float64[m],
    d_neff int64[m] (or None), d_best_status int32[2] -> (best, status)."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    for t, name in ((d_x, "x"), (d_y, "y"), (d_h, "h"), (d_cv, "cv")):
        if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
            raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if d_cv.numel() != m or d_best_status.numel() != 2 or d_best_status.dtype != torch.int32:
        raise ValueError("cv must have m elements, best_status 2 int32")
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    st = _lib().kr_cv_grid_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                 _algo_id(algo), d_cv.data_ptr(), None if d_neff is None else d_neff.data_ptr(),
                                 d_best_status.data_ptr(), d_ws.data_ptr(), d_ws.numel() * d_ws.element_size(),
                                 ctypes.c_void_p(s.cuda_stream))
    _check(st, "kr_cv_grid_async")


def kr_finalize_async(d_partial, n: int, m: int, d_cv, d_neff, d_best_status, stream=None) -> None:
    """Device finalize: d_cv float64[m], d_neff int64[m] (or None),
    d_best_status int32[2] -> (best, status)."""
    import torch

    _check_f64("partial", d_partial, partial_len(m))
    _check_f64("cv", d_cv, m)
    _check_neff(d_neff, m)
    _check_best_status(d_best_status)
    s = torch.cuda.current_stream(d_partial.device) if stream is None else stream
    st = _lib().kr_finalize_async(d_partial.data_ptr(), int(n), int(m), d_cv.data_ptr(),
                                  None if d_neff is None else d_neff.data_ptr(),
                                  d_best_status.data_ptr(), d_best_status.data_ptr() + 4,
                                  ctypes.c_void_p(s.cuda_stream))
    _check(st, "kr_finalize_async")


_PROFILING = {"on": False}


def kr_profile_enable(on: bool) -> None:
    _lib().kr_profile_enable(1 if on else 0)
    _PROFILING["on"] = bool(on)


def kr_profile_enabled() -> bool:
    """Whether kr_profile_enable(True) is in effect (as set through this binding)."""
    return _PROFILING["on"]


def kr_profile_read():
    """(sort_ms, prefix_build_ms, sweep_ms, reduce_ms) of the last
    kr_cv_shard_async on this thread."""
    ms = np.zeros(4, np.float32)
    _check(_lib().kr_profile_read(ms.ctypes.data), "kr_profile_read")
    return tuple(float(v) for v in ms)


def kr_last_algo() -> int:
    return int(_lib().kr_last_algo())


def kr_launch_count() -> int:
    return int(_lib().kr_launch_count())


def workspace(n: int, m: int, device=None, kernel=None, algo=None, kde: bool = False):
    """A device workspace tensor (PyTorch caching allocator; take aligned()).
    Sized for every entry point unless algo (with kernel) or kde narrows it."""
    import torch

    nbytes = kr_workspace_bytes(n, m, kernel, algo, kde)
    if nbytes == 0:
        raise KrcvError(KR_ECUDA, "kr_workspace_bytes")
    return torch.empty(nbytes + 256, dtype=torch.uint8, device=device)


def aligned(ws):
    """View of ws starting at a 256-byte boundary."""
    off = (-ws.data_ptr()) % 256
    return ws[off:]


# ------------------------------------------------------------ KDE (LSCV, Q24)
def kr_kde_lscv(x, h, kernel="epanechnikov"):
    """KDE least-squares CV on the current CUDA device: (lscv[m], best)."""
    x, h = _host(x), _host(h)
    m = h.shape[0]
    out = np.empty(m, np.float64)
    best = ctypes.c_int32(-1)
    _check(_lib().kr_kde_lscv(x.ctypes.data, x.shape[0], h.ctypes.data, m, _kernel_id(kernel), out.ctypes.data,
                              ctypes.byref(best)), "kr_kde_lscv")
    return out, int(best.value)


def kr_kde_shard_async(d_x, d_h, kernel, shard: int, nshards: int, d_partial, d_ws, stream=None) -> None:
    """Enqueue one row shard of the KDE LSCV -> partial [sum A | sum B | status]."""
    import torch

    _check_f64("x", d_x)
    _check_f64("h", d_h)
    _check_f64("partial", d_partial, partial_len(d_h.numel()))
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    _check(_lib().kr_kde_shard_async(d_x.data_ptr(), d_x.numel(), d_h.data_ptr(), d_h.numel(), _kernel_id(kernel),
                                     int(shard), int(nshards), d_partial.data_ptr(), d_ws.data_ptr(),
                                     d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream)),
           "kr_kde_shard_async")


def kr_kde_finalize(partial, n: int, h, kernel="epanechnikov"):
    p, h = _host(partial), _host(h)
    if p.shape[0] != partial_len(h.shape[0]):
        raise ValueError("partial must have length 2m+2")
    out = np.empty(h.shape[0], np.float64)
    best = ctypes.c_int32(-1)
    _check(_lib().kr_kde_finalize(p.ctypes.data, int(n), h.ctypes.data, h.shape[0], _kernel_id(kernel),
                                  out.ctypes.data, ctypes.byref(best)), "kr_kde_finalize")
    return out, int(best.value)


# ------------------------------------------------------- local-linear (Q25)
def kr_ll_cv_grid(x, y, h, kernel="epanechnikov", with_neff: bool = False):
    """Local-linear LOO-CV grid search from host arrays (kr_ll_cv_grid).
    Returns (cv[m], best) or (cv, neff, best)."""
    x, y, h = _host(x), _host(y), _host(h)
    if x.shape != y.shape or x.ndim != 1:
        raise ValueError("x and y must be 1-D arrays of equal length")
    n, m = x.shape[0], h.shape[0]
    cv = np.empty(m, np.float64)
    neff = np.empty(m, np.int64)
    best = ctypes.c_int32(-1)
    _check(_lib().kr_ll_cv_grid(x.ctypes.data, y.ctypes.data, n, h.ctypes.data, m, _kernel_id(kernel),
                                cv.ctypes.data, neff.ctypes.data, ctypes.byref(best)), "kr_ll_cv_grid")
    return (cv, neff, int(best.value)) if with_neff else (cv, int(best.value))


def kr_ll_cv_grid_async(d_x, d_y, d_h, kernel, d_cv, d_neff, d_best_status, d_ws, stream=None) -> None:
    """Enqueue the whole single-GPU local-linear search (tensors as kr_cv_grid_async)."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    for t, name in ((d_x, "x"), (d_y, "y"), (d_h, "h"), (d_cv, "cv")):
        if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
            raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if d_cv.numel() != m or d_best_status.numel() != 2 or d_best_status.dtype != torch.int32:
        raise ValueError("cv must have m elements, best_status 2 int32")
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    _check(_lib().kr_ll_cv_grid_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                      d_cv.data_ptr(), None if d_neff is None else d_neff.data_ptr(),
                                      d_best_status.data_ptr(), d_ws.data_ptr(), d_ws.numel() * d_ws.element_size(),
                                      ctypes.c_void_p(s.cuda_stream)), "kr_ll_cv_grid_async")


def kr_ll_shard_async(d_x, d_y, d_h, kernel, shard: int, nshards: int, d_partial, d_ws, stream=None) -> None:
    """Enqueue one row shard of the local-linear search -> additive partial
    [S | neff | status] (finalize with kr_finalize / kr_finalize_async)."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    for t, name in ((d_x, "x"), (d_y, "y"), (d_h, "h"), (d_partial, "partial")):
        if not (t.is_cuda and t.dtype == torch.float64 and t.is_contiguous()):
            raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if d_partial.numel() != partial_len(m):
        raise ValueError("partial must have 2m+2 elements")
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    _check(_lib().kr_ll_shard_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                    int(shard), int(nshards), d_partial.data_ptr(), d_ws.data_ptr(),
                                    d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream)),
           "kr_ll_shard_async")


# ------------------------------------- LOO confidence intervals (Q26)
def kr_cv_ci(x, y, h, kernel="epanechnikov"):
    """Grid search, then at the CV-optimal bandwidth the Nadaraya-Watson
    estimate and its delete-one jackknife standard error at every observation
    (reading Q26): (cv[m], est[n], se[n], best).  se is NaN where a point's
    window holds only itself."""
    x, y, h = _host(x), _host(y), _host(h)
    if x.shape != y.shape or x.ndim != 1:
        raise ValueError("x and y must be 1-D arrays of equal length")
    n, m = x.shape[0], h.shape[0]
    cv, est, se = np.empty(m), np.empty(n), np.empty(n)
    best = ctypes.c_int32(-1)
    _check(_lib().kr_cv_ci(x.ctypes.data, y.ctypes.data, n, h.ctypes.data, m, _kernel_id(kernel), cv.ctypes.data,
                           est.ctypes.data, se.ctypes.data, ctypes.byref(best)), "kr_cv_ci")
    return cv, est, se, int(best.value)


def kr_kde_ci(x, h, kernel="epanechnikov"):
    """KDE LSCV grid search, then at the optimal bandwidth the density estimate
    and its delete-one jackknife standard error at every observation
    (reading Q26): (lscv[m], est[n], se[n], best)."""
    x, h = _host(x), _host(h)
    n, m = x.shape[0], h.shape[0]
    lscv, est, se = np.empty(m), np.empty(n), np.empty(n)
    best = ctypes.c_int32(-1)
    _check(_lib().kr_kde_ci(x.ctypes.data, n, h.ctypes.data, m, _kernel_id(kernel), lscv.ctypes.data,
                            est.ctypes.data, se.ctypes.data, ctypes.byref(best)), "kr_kde_ci")
    return lscv, est, se, int(best.value)


def kr_cv_ci_async(d_x, d_y, d_h, kernel, d_cv, d_est, d_se, d_best_status, d_ws, stream=None) -> None:
    """Device form of kr_cv_ci (CUDA tensors; enqueued on `stream`)."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    for t, name in ((d_x, "x"), (d_y, "y"), (d_h, "h")):
        _check_f64(name, t)
    _check_f64("y", d_y, n)
    _check_f64("cv", d_cv, m)
    _check_f64("est", d_est, n)
    _check_f64("se", d_se, n)
    _check_best_status(d_best_status)
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    _check(_lib().kr_cv_ci_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel),
                                 d_cv.data_ptr(), d_est.data_ptr(), d_se.data_ptr(), d_best_status.data_ptr(),
                                 d_ws.data_ptr(), d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream)),
           "kr_cv_ci_async")


def kr_kde_ci_async(d_x, d_h, kernel, d_lscv, d_est, d_se, d_best_status, d_ws, stream=None) -> None:
    """Device form of kr_kde_ci (CUDA tensors; enqueued on `stream`)."""
    import torch

    n, m = d_x.numel(), d_h.numel()
    _check_f64("x", d_x)
    _check_f64("h", d_h)
    _check_f64("lscv", d_lscv, m)
    _check_f64("est", d_est, n)
    _check_f64("se", d_se, n)
    _check_best_status(d_best_status)
    s = torch.cuda.current_stream(d_x.device) if stream is None else stream
    _check(_lib().kr_kde_ci_async(d_x.data_ptr(), n, d_h.data_ptr(), m, _kernel_id(kernel), d_lscv.data_ptr(),
                                  d_est.data_ptr(), d_se.data_ptr(), d_best_status.data_ptr(), d_ws.data_ptr(),
                                  d_ws.numel() * d_ws.element_size(), ctypes.c_void_p(s.cuda_stream)),
           "kr_kde_ci_async")


def confidence_intervals(est, se, level: float = 0.95):
    """(lo, hi) = est -+ z se with z = Phi^-1((1 + level) / 2) (arithmetic on
    the outputs of kr_cv_ci / kr_kde_ci; no device work)."""
    from statistics import NormalDist

    z = NormalDist().inv_cdf(0.5 + 0.5 * float(level))
    est, se = np.asarray(est, np.float64), np.asarray(se, np.float64)
    return est - z * se, est + z * se
