"""Load balance of the row sharding: on one GPU, run every
shard r of P (kr_cv_shard_async, the multi-GPU code path of one rank) and
time its window kernel with the library's stage events; prints the max/mean
ratio per (config, P) -- the factor by which the slowest rank would stretch
a P-GPU step -- for equal-row shards and for the cost-balanced cuts
GridSearch(balance=True) derives (api.balanced_cuts over 4 P timed
segments).  python tools/shard_balance.py [C3 C4 C5]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads  # noqa: E402
from paper_conf_ipps_rohlfsz17_b200 import krcv  # noqa: E402
from paper_conf_ipps_rohlfsz17_b200.api import balanced_cuts  # noqa: E402


def window_ms(d_x, d_y, d_h, k, lo, hi, part, ws):
    krcv.kr_profile_enable(True)
    for _ in range(3):
        krcv.kr_cv_rows_async(d_x, d_y, d_h, k, lo, hi, part, ws)
        ms = krcv.kr_profile_read()[2]
    krcv.kr_profile_enable(False)
    return ms


def main(cfgs):
    dev = torch.device("cuda", 0)
    for c in cfgs:
        x, y, h, k = workloads.make(c, seed=0)
        n, m = x.shape[0], h.shape[0]
        d_x, d_y, d_h = (torch.as_tensor(v, device=dev) for v in (x, y, h))
        ws = krcv.aligned(krcv.workspace(n, m, dev))
        part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device=dev)
        for P in (2, 4, 8):
            eq = np.array([window_ms(d_x, d_y, d_h, k, (r * n) // P, ((r + 1) * n) // P, part, ws) for r in range(P)])
            S = 4 * P
            cost = [window_ms(d_x, d_y, d_h, k, (s * n) // S, ((s + 1) * n) // S, part, ws) for s in range(S)]
            cuts = balanced_cuts(cost, n, P)
            bal = np.array([window_ms(d_x, d_y, d_h, k, a, b, part, ws) for a, b in zip(cuts, cuts[1:])])
            print(f"{c} P={P}: equal rows max/mean {eq.max() / eq.mean():.3f} (max {eq.max():.3f} ms); "
                  f"balanced max/mean {bal.max() / bal.mean():.3f} (max {bal.max():.3f} ms); "
                  f"slowest rank {eq.max() / bal.max():.3f}x faster", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C3", "C4", "C5"])
