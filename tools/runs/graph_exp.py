"""Experiment: device time of one C2 grid search launched directly vs replayed
from a CUDA graph captured around GridSearch.run (same stream, L2 flushed)."""
import json, sys, time
import torch
sys.path.insert(0, ".")
import workloads
from paper_conf_ipps_rohlfsz17_b200.api import GridSearch

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
x, y, h, k = workloads.make(cfg, seed=0)
n, m = x.shape[0], h.shape[0]
dev = torch.device("cuda", 0)
d_x, d_y = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
plan = GridSearch(n, h, k, device=dev)
s = torch.cuda.Stream()
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
with torch.cuda.stream(s):
    for _ in range(5):
        plan.run(d_x, d_y)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan.run(d_x, d_y)
    torch.cuda.synchronize()
    out = {}
    for mode in ("direct", "graph", "direct", "graph"):
        ts = []
        for i in range(30):
            flush.fill_(i & 255)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            if mode == "graph":
                g.replay()
            else:
                plan.run(d_x, d_y)
            b.record(s)
            b.synchronize()
            ts.append(a.elapsed_time(b))
        ts.sort()
        out[mode] = {"median_ms": ts[len(ts) // 2], "min_ms": ts[0]}
    r = plan.result()
    out["best"] = r.best
print(json.dumps({"config": cfg, **out}))
