"""Measured table for BASELINE.md §6 (run on the GPU box): for C1-C5 x seeds
0-2, the device time of one full grid search (CUDA-graph replay, x/y
resident, L2 flushed between steps, median of 10 after 3 warm-ups), the
end-to-end time through kr_cv_grid from pinned host buffers (median of 10),
pair-bandwidth evaluations per second, and parity against the oracle's
curves (tests/golden/curves/, written from oracle/ only).  Prints a markdown
table and writes it to the path given (default gpurun_out/parity_report.md).
"""
import ctypes
import glob
import os
import statistics
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import workloads  # noqa: E402
from paper_conf_ipps_rohlfsz17_b200 import krcv  # noqa: E402
from paper_conf_ipps_rohlfsz17_b200.api import GridSearch  # noqa: E402
from tests.helpers import best_ok, cv_rel_err  # noqa: E402


def main(out_path):
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    rows = ["| config | seed | n | m | device ms | e2e ms | pair·bw/s | max rel err vs oracle | best (oracle) | n_eff equal |",
            "|---|---|---|---|---|---|---|---|---|---|"]
    for path in sorted(glob.glob(os.path.join(ROOT, "tests", "golden", "curves", "C*_s*.npz"))):
        cfg, seed = os.path.basename(path)[:-4].split("_s")
        ref = np.load(path)
        x, y, h, k = workloads.make(cfg, seed=int(seed))
        n, m = x.shape[0], h.shape[0]
        d_x, d_y = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
        plan = GridSearch(n, h, k, device=dev, graph=True)
        for _ in range(3):
            plan.run(d_x, d_y)
        torch.cuda.synchronize()
        ts = []
        for s in range(10):
            flush.fill_(s)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            plan.run(d_x, d_y)
            b.record()
            b.synchronize()
            ts.append(a.elapsed_time(b))
        res = plan.result()
        cv, neff = res.cv.cpu().numpy(), res.neff.cpu().numpy()
        hx, hy, hh = (torch.from_numpy(v).pin_memory() for v in (x, y, h))
        hcv = torch.empty(m, dtype=torch.float64).pin_memory()
        best = ctypes.c_int32(-1)
        we = []
        for s in range(13):
            t0 = time.perf_counter()
            st = krcv.kr_cv_grid_ptr(hx.data_ptr(), hy.data_ptr(), n, hh.data_ptr(), m, k, hcv.data_ptr(),
                                     ctypes.byref(best))
            t1 = time.perf_counter()
            assert st == 0
            if s >= 3:
                we.append((t1 - t0) * 1e3)
        assert np.array_equal(hcv.numpy().view(np.uint64), cv.view(np.uint64))  # host API = device plan
        td, tw = statistics.median(ts), statistics.median(we)
        err = cv_rel_err(cv, ref["cv"])
        ok = best_ok(res.best, ref["cv"], 1e-6)
        rows.append(f"| {cfg} | {seed} | {n:,} | {m} | {td:.4g} | {tw:.4g} | {n * (n - 1) * m / (td * 1e-3):.3g} | "
                    f"{err:.2g} | {res.best} ({int(ref['best'])}){'' if ok else ' MISMATCH'} | "
                    f"{'yes' if np.array_equal(neff, ref['neff']) else 'NO'} |")
        print(rows[-1], flush=True)
        del plan
        torch.cuda.empty_cache()
    text = "\n".join(rows) + "\n"
    with open(out_path, "w") as f:
        f.write(text)
    print(text)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "parity_report.md"))
