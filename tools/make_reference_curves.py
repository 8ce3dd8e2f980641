"""Reference CV curves for the full BASELINE.json configurations (C1-C5,
seeds 0-2), written by the oracle only (tests/golden/curves/<C>_s<seed>.npz:
cv, neff, best, and which evaluator).  C1, C2, C3, C5: the oracle's
Program-3 evaluator (kro_cv_sorted, long double; PAPER.md P@27643, Program 3
"Sequential C"), with the oracle's independent window-prefix checker
(oracle/window.py, numpy long double, exact Q1 membership predicate) stored
beside it for C3 and C5 as a second evaluator (cv_window, neff_window) and
their agreement recorded.  C4: the window checker only (Program 3 would cost
~1.4e5 core-seconds); tests/test_gpu_parity.py checks C4
row shards against Program 3 directly.  Inputs come from workloads/ (seeded
generators, no method arithmetic).  tests/test_gpu_baseline_curves.py
compares the CUDA path, in the launch configuration bench.py times, against
these.

    python tools/make_reference_curves.py [--force] [C1 C2 ...]
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


PROGRAM3 = ("C1", "C2", "C3", "C5")


def main(cfgs, force=False):
    os.makedirs(OUT, exist_ok=True)
    for c in cfgs:
        for seed in (0, 1, 2):
            path = os.path.join(OUT, f"{c}_s{seed}.npz")
            if os.path.exists(path) and not force:
                continue
            x, y, h, k = workloads.make(c, seed=seed)
            t = time.time()
            extra = {}
            if c in PROGRAM3:
                r = oracle.cv_sorted(x, y, h, k)
                cv, neff, best, how = r.cv, r.neff, r.best, "oracle.cv_sorted (kro_cv_sorted, long double)"
                if c in ("C3", "C5"):
                    w = window.cv_window(x, y, h, k)
                    cvw = np.asarray(w["cv"], np.float64)
                    floor = 1e-12 * float(np.max(np.abs(cv)))
                    agree = float(np.max(np.abs(cvw - cv) / np.maximum(np.abs(cv), floor)))
                    extra = dict(cv_window=cvw, neff_window=np.asarray(w["neff"], np.int64),
                                 best_window=int(w["best"]), window_vs_program3=agree)
            else:
                r = window.cv_window(x, y, h, k)
                cv, neff, best, how = r["cv"], r["neff"], r["best"], "oracle.window.cv_window (numpy long double)"
            np.savez(path, cv=np.asarray(cv, np.float64), neff=np.asarray(neff, np.int64), best=int(best),
                     evaluator=how, n=x.shape[0], m=h.shape[0], kernel=int(k), seed=seed, **extra)
            note = f", window checker vs Program 3 {extra['window_vs_program3']:.2e}" if extra else ""
            print(f"{c} seed {seed}: best {best} cv {cv[best]:.12g} ({time.time() - t:.1f} s, {how}{note})",
                  flush=True)


if __name__ == "__main__":
    args = [a for a in sys.argv[1:] if a != "--force"]
    main(args or ["C1", "C2", "C3", "C5", "C4"], force="--force" in sys.argv[1:])
