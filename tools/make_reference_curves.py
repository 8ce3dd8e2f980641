"""Reference CV curves for the full BASELINE.json configurations (C1-C5,
seeds 0-2), written by the oracle only (tests/golden/curves/<C>_s<seed>.npz:
cv, neff, best, and which evaluator).  C1, C2: the oracle's Program-3
evaluator (kro_cv_sorted, long double).  C3, C4, C5: the oracle's
independent window-prefix checker (oracle/window.py, numpy long double with
the exact Q1 membership predicate; pinned against kro_cv_sorted at <= 1e-12
for Epanechnikov, P10).  Inputs come from workloads/ (seeded generators, no
method arithmetic).  tests/test_gpu_baseline_curves.py compares the CUDA
path, in the launch configuration bench.py times, against these.

    python tools/make_reference_curves.py [C1 C2 ...]
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import workloads  # noqa: E402
from oracle import window  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "curves")


def main(cfgs):
    os.makedirs(OUT, exist_ok=True)
    for c in cfgs:
        for seed in (0, 1, 2):
            path = os.path.join(OUT, f"{c}_s{seed}.npz")
            if os.path.exists(path):
                continue
            x, y, h, k = workloads.make(c, seed=seed)
            t = time.time()
            if c in ("C1", "C2"):
                r = oracle.cv_sorted(x, y, h, k)
                cv, neff, best, how = r.cv, r.neff, r.best, "oracle.cv_sorted (kro_cv_sorted, long double)"
            else:
                r = window.cv_window(x, y, h, k)
                cv, neff, best, how = r["cv"], r["neff"], r["best"], "oracle.window.cv_window (numpy long double)"
            np.savez(path, cv=np.asarray(cv, np.float64), neff=np.asarray(neff, np.int64), best=int(best),
                     evaluator=how, n=x.shape[0], m=h.shape[0], kernel=int(k), seed=seed)
            print(f"{c} seed {seed}: best {best} cv {cv[best]:.12g} ({time.time() - t:.1f} s, {how})", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C1", "C2", "C3", "C5", "C4"])
