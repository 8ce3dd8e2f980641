"""Load balance of the row sharding: on one GPU, run every
shard r of P (kr_cv_shard_async, the multi-GPU code path of one rank) and
time its window kernel with the library's stage events; prints the max/mean
ratio per (config, P) -- the factor by which the slowest rank would stretch
a P-GPU step.  python tools/shard_balance.py [C3 C4 C5]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads  # noqa: E402
from paper_conf_ipps_rohlfsz17_b200 import krcv  # noqa: E402


def main(cfgs):
    dev = torch.device("cuda", 0)
    for c in cfgs:
        x, y, h, k = workloads.make(c, seed=0)
        n, m = x.shape[0], h.shape[0]
        d_x, d_y, d_h = (torch.as_tensor(v, device=dev) for v in (x, y, h))
        ws = krcv.aligned(krcv.workspace(n, m, dev))
        part = torch.empty(krcv.partial_len(m), dtype=torch.float64, device=dev)
        for P in (2, 4, 8):
            t = []
            for r in range(P):
                krcv.kr_profile_enable(True)
                for rep in range(3):
                    krcv.kr_cv_shard_async(d_x, d_y, d_h, k, r, P, part, ws)
                    ms = krcv.kr_profile_read()
                krcv.kr_profile_enable(False)
                t.append(ms[2])
            t = np.array(t)
            print(f"{c} P={P}: window ms per shard {np.round(t, 3).tolist()}  max/mean {t.max() / t.mean():.3f}",
                  flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C3", "C4", "C5"])
