"""The row-sharded multi-rank device path on one GPU: 2 and 3 processes
(torch.multiprocessing, gloo backend -- NCCL refuses two ranks on one device)
all on cuda:0, each running its shard through the C-ABI device entry points,
the all-reduce of the 2m+2 partial vector and the device finalize
(api.GridSearch with world > 1).  Every rank must return the single-GPU
answer (CV to 1e-12: the shard partials add in another order; n_eff and best
exact) and the oracle's."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, cfg, n, estimator, algo, q, balance=False):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import workloads
        from paper_conf_ipps_rohlfsz17_b200 import api

        torch.cuda.set_device(0)
        x, y, h, k = workloads.make(cfg, seed=6, n=n)
        r = api.cv_grid(x, y, h, kernel=k, distributed=True, algo=algo, estimator=estimator, balance=balance)
        q.put((rank, r.cv.cpu().numpy(), r.neff.cpu().numpy(), r.best))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg,n,estimator,algo,balance", [
    (2, "C2", 3000, "nw", "auto", False),
    (3, "C5", 2500, "nw", "auto", False),
    (2, "C2", 3000, "nw", "sweep", False),
    (2, "C1", 1000, "nw", "hist", False),
    (3, "C2", 2000, "ll", "auto", False),
    (3, "C5", 2500, "nw", "auto", True),    # cost-balanced cuts (rank 0 calibrates, broadcast)
    (2, "C2", 3000, "nw", "sweep", True),
])
def test_sharded_device_path_matches_single_gpu(world, cfg, n, estimator, algo, balance):
    import oracle
    import workloads
    from paper_conf_ipps_rohlfsz17_b200 import api
    from tests.helpers import best_ok, cv_rel_err

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, n, estimator, algo, q, balance))
             for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    x, y, h, k = workloads.make(cfg, seed=6, n=n)
    single = api.cv_grid(x, y, h, kernel=k, algo=algo, estimator=estimator)
    ref = oracle.ll_cv(x, y, h, k) if estimator == "ll" else oracle.cv_sorted(x, y, h, k)
    for rank, cv, neff, best in res:
        assert cv_rel_err(cv, single.cv.cpu().numpy()) <= 1e-12
        assert np.array_equal(neff, single.neff.cpu().numpy())
        assert best == single.best
        assert cv_rel_err(cv, ref.cv) <= 1e-10 and np.array_equal(neff, ref.neff) and best_ok(best, ref.cv)
    assert all(np.array_equal(r[1], res[0][1]) and r[3] == res[0][3] for r in res)
