"""Where the end-to-end time of kr_cv_grid goes (host arrays in pinned
memory -> results on the host): for several n at m = 200, the device time of
the same search (graph replay, x/y resident) and the end-to-end time; their
difference is the host-call overhead (graph launch, H2D of 16n + 8m bytes,
D2H of 16m + 8 bytes, synchronisation)."""
import ctypes
import os
import statistics
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rohlfsz17_b200 import krcv  # noqa: E402
from paper_conf_ipps_rohlfsz17_b200.api import GridSearch  # noqa: E402

dev = torch.device("cuda", 0)
rng = np.random.default_rng(0)
for n in (2, 1000, 20000, 100000):
    m = 200
    x = rng.uniform(0, 1, n)
    y = 0.5 * x + 10 * x * x + rng.uniform(0, 0.5, n)
    h = krcv.kr_default_grid(x, m) if n > 2 else np.linspace(0.5, 1.0, m)
    d_x, d_y = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
    plan = GridSearch(n, h, 1, device=dev, graph=True)
    for _ in range(3):
        plan.run(d_x, d_y)
    torch.cuda.synchronize()
    ts = []
    for _ in range(20):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); plan.run(d_x, d_y); b.record(); b.synchronize()
        ts.append(a.elapsed_time(b))
    hx, hy, hh = (torch.from_numpy(v).pin_memory() for v in (x, y, h))
    hcv = torch.empty(m, dtype=torch.float64).pin_memory()
    best = ctypes.c_int32(-1)
    we = []
    for s in range(23):
        t0 = time.perf_counter()
        krcv.kr_cv_grid_ptr(hx.data_ptr(), hy.data_ptr(), n, hh.data_ptr(), m, 1, hcv.data_ptr(), ctypes.byref(best))
        t1 = time.perf_counter()
        if s >= 3:
            we.append((t1 - t0) * 1e3)
    td, tw = statistics.median(ts), statistics.median(we)
    print(f"n={n:7d} m={m}: device {td * 1e3:8.1f} us  e2e {tw * 1e3:8.1f} us  overhead {1e3 * (tw - td):6.1f} us "
          f"(H2D {16 * n + 8 * m} B)", flush=True)
