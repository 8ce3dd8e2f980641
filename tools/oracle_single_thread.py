#!/usr/bin/env python
"""One-thread time of the oracle's Program-3 evaluator (kro_cv_sorted) on C1
and C2, next to the paper's Table I figure for its own sequential C program
at n = 20,000, k = 50: 80.92 s (PAPER.md P@33218; VERDICT r01 "record the
1-thread oracle time").  Run with OMP_NUM_THREADS=1 (set here before the
oracle library loads).

    python tools/oracle_single_thread.py [--out profiles/oracle_single_thread.json]
"""
import argparse
import json
import os
import platform
import sys
import time

os.environ["OMP_NUM_THREADS"] = "1"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import workloads  # noqa: E402


def cpu_model():
    for line in open("/proc/cpuinfo"):
        if line.startswith("model name"):
            return line.split(":", 1)[1].strip()
    return platform.processor()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    assert oracle.num_threads() == 1, oracle.num_threads()
    res = {"cpu": cpu_model(), "threads": 1, "evaluator": "oracle.cv_sorted (kro_cv_sorted, long double)",
           "paper_table_I": {"n": 20000, "k": 50, "sequential_C_s": 80.92, "cite": "PAPER.md P@33218"},
           "runs": []}
    for cfg, m in (("C1", None), ("C2", 50), ("C2", None)):
        x, y, h, k = workloads.make(cfg, seed=0)
        if m is not None:  # the paper's k = 50 on C2's data: its default grid with 50 points
            h = workloads.grid_default(x, m)
        t = time.perf_counter()
        r = oracle.cv_sorted(x, y, h, k)
        dt = time.perf_counter() - t
        res["runs"].append({"config": cfg, "n": int(x.shape[0]), "m": int(h.shape[0]), "kernel": int(k),
                            "seconds": dt, "best": int(r.best)})
        print(json.dumps(res["runs"][-1]), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
