"""Multi-process host logic of the row-sharded path on CPU (gloo, world
size 2 and 3): each rank computes its shard's partial vector -- here with the
oracle's shard mode standing in for the GPU shard call -- then the product's
all-reduce + finalize (api.allreduce_partial / api.finalize_partial, the
C-ABI host kr_finalize) must reproduce the unsharded oracle result on every
rank."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, cfg, n, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import workloads
        from paper_conf_ipps_rohlfsz17_b200 import api

        x, y, h, k = workloads.make(cfg, seed=rank * 0 + 4, n=n)  # identical inputs on every rank
        m = h.shape[0]
        lo, hi = api.shard_bounds(n, rank, world)
        rows = oracle.sorted_rows(x)[lo:hi]
        assert np.array_equal(rows, oracle.shard_rows(x, rank, world))
        part = oracle.cv_sorted(x, y, h, k, rows=rows) if rows.size else None
        partial = torch.zeros(2 * m + 2, dtype=torch.float64)
        if part is not None:
            partial[:m] = torch.from_numpy(part.S)
            partial[m:2 * m] = torch.from_numpy(part.neff.astype(np.float64))
        api.allreduce_partial(partial)
        cv, neff, best = api.finalize_partial(partial, n, m)
        q.put((rank, cv.numpy(), neff.numpy(), best))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg,n", [(2, "C2", 600), (3, "C5", 500), (2, "C1", 5)])
def test_sharded_allreduce_matches_unsharded(world, cfg, n):
    import oracle
    import workloads
    from tests.helpers import best_ok, cv_rel_err

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, cfg, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    x, y, h, k = workloads.make(cfg, seed=4, n=n)
    ref = oracle.cv_sorted(x, y, h, k)
    for rank, cv, neff, best in res:
        assert cv_rel_err(cv, ref.cv) <= 1e-14
        assert np.array_equal(neff, ref.neff)
        assert best_ok(best, ref.cv)
    # every rank returns the identical answer
    assert all(np.array_equal(r[1], res[0][1]) and r[3] == res[0][3] for r in res)


def test_shard_bounds_partition():
    from paper_conf_ipps_rohlfsz17_b200 import api

    for n in (2, 3, 7, 1000, 20001):
        for P in (1, 2, 3, 8, 64):
            b = [api.shard_bounds(n, r, P) for r in range(P)]
            assert b[0][0] == 0 and b[-1][1] == n
            assert all(b[i][1] == b[i + 1][0] for i in range(P - 1))
            assert all(hi - lo in (n // P, n // P + 1) for lo, hi in b)
    with pytest.raises(ValueError):
        api.shard_bounds(10, 2, 2)


# ------------------------------------------------------------ balanced cuts
def test_balanced_cuts_uniform_cost_is_equal_rows():
    from paper_conf_ipps_rohlfsz17_b200.api import balanced_cuts
    cuts = balanced_cuts(np.ones(32), 64 * 1000, 8)
    assert cuts == [r * 8000 for r in range(9)]


def test_balanced_cuts_equalise_skewed_cost():
    """A slow tail (the C5 shape) moves the cuts so every rank's share of the
    cost is within one alignment block of 1/P, and the cuts tile [0, n)."""
    from paper_conf_ipps_rohlfsz17_b200.api import balanced_cuts
    rng = np.random.default_rng(3)
    S, n, P = 128, 1_000_000, 8
    cost = 1.0 + rng.uniform(0, 0.2, S)
    cost[-8:] *= 4.0
    cuts = balanced_cuts(cost, n, P)
    assert cuts[0] == 0 and cuts[-1] == n and all(a <= b for a, b in zip(cuts, cuts[1:]))
    assert all(c % 64 == 0 for c in cuts[1:-1])
    # per-row cost, piecewise constant over the segments
    bounds = [(s * n) // S for s in range(S + 1)]
    row_cost = np.repeat(cost / np.diff(bounds), np.diff(bounds))
    share = np.array([row_cost[a:b].sum() for a, b in zip(cuts, cuts[1:])]) / row_cost.sum()
    assert np.max(np.abs(share - 1.0 / P)) <= 64 * row_cost.max() / row_cost.sum() + 1e-12
    equal = np.array([row_cost[(r * n) // P:((r + 1) * n) // P].sum() for r in range(P)]) / row_cost.sum()
    assert share.max() < equal.max()


def test_balanced_cuts_degenerate_inputs():
    from paper_conf_ipps_rohlfsz17_b200.api import balanced_cuts
    assert balanced_cuts(np.zeros(16), 1000, 4) == [0, 250, 500, 750, 1000]   # no cost measured
    assert balanced_cuts(np.ones(16), 1000, 1) == [0, 1000]
    cuts = balanced_cuts(np.r_[np.zeros(15), 1.0], 100, 4)                   # all cost in the last segment
    assert cuts[0] == 0 and cuts[-1] == 100 and all(a <= b for a, b in zip(cuts, cuts[1:]))
