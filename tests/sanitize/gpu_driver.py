"""T7 device half: run every CUDA path once at small sizes
so that compute-sanitizer (memcheck / racecheck / synccheck / initcheck) sees
every kernel: the chunked rank sort and the CUB onesweep sort, the prefix
build (two-phase, fused with its grid barrier, one-CTA), the bucket table,
the window kernel (KRCV_WIN=r01 selects r01's), the per-pair sweep, the
histogram ordering, the dense Gaussian kernel, KDE LSCV, local-linear CV,
the leave-one-out confidence intervals, refinement, the reduction with its
fused finalize, and the shard + finalize path.  Host arrays only (no torch kernels in the trace).  Test
infrastructure: called by tests/test_gpu_sanitizer.py."""
import sys

import numpy as np

from paper_conf_ipps_rohlfsz17_b200 import krcv


def main() -> int:
    rng = np.random.default_rng(3)
    small = int(sys.argv[1]) if len(sys.argv) > 1 else 700
    x = np.floor(rng.uniform(0, 256, small)) / 64.0  # dyadic: duplicates and exact distances
    y = np.sin(x) + rng.normal(0, 0.5, small)
    h = np.concatenate([krcv.kr_default_grid(x, 10), [0.25, 0.25]])
    h.sort()
    for k in ("uniform", "epanechnikov", "triangular"):
        for algo in ("sweep", "prefix", "hist"):
            cv, best = krcv.kr_cv_grid(x, y, h, k, algo=algo)
            assert 0 <= best < h.size and np.all(np.isfinite(cv))
        krcv.kr_cv_refine(x, y, h, k, levels=2, m_fine=9)
        krcv.kr_kde_lscv(x, h, k)
        krcv.kr_ll_cv_grid(x, y, h, k)
        krcv.kr_cv_ci(x, y, h, k)
        krcv.kr_kde_ci(x, h, k)
    # the fused O(n) build (n > 1,024 and <= 148 x 256) and the two-phase one above it
    for nn in (5_000, 60_000):
        xm = rng.uniform(0, 1, nn)
        ym = xm + rng.normal(0, 0.1, nn)
        krcv.kr_cv_grid(xm, ym, np.linspace(0.001, 1.0, 7), "epanechnikov", algo="prefix")
    krcv.kr_cv_grid(x, y, h, "gaussian")
    krcv.kr_cv_grid(x[:2], y[:2], h, "epanechnikov")  # n = 2
    # CUB onesweep sort path (n > 131,072), window-prefix only (the sweep is O(n^2))
    xl = rng.lognormal(0.0, 1.0, 140_000)
    yl = np.sin(xl) + rng.normal(0, 0.5, xl.size)
    hl = np.geomspace(1e-3, xl.max() - xl.min(), 6)
    krcv.kr_cv_grid(xl, yl, hl, "epanechnikov", algo="prefix")
    # error path: non-finite input reported, outputs untouched
    xb = x.copy()
    xb[5] = np.nan
    try:
        krcv.kr_cv_grid(xb, y, h, "epanechnikov")
        return 2
    except krcv.KrcvError:
        pass
    krcv.kr_release()  # the per-device host-call state: memcheck --leak-check sees it freed
    print("gpu sanitizer driver: ok")
    return 0


if __name__ == "__main__":
    sys.exit(main())
