"""Python-level API over the C-ABI: single- and multi-GPU grid search.

PyTorch supplies device memory (caching allocator), streams and the process
group; the computation is the C-ABI's (libkrcv.so).  Row sharding follows
SURVEY.md §8(e): rank r of P sweeps sorted rows [floor(r n/P), floor((r+1) n/P)),
then ONE all-reduce(SUM) of the partial vector [S | neff | status] (2m+2
fp64) over NCCL, then every rank finalizes identically on its device.
"""
from __future__ import annotations

import dataclasses

import numpy as np

from . import krcv


@dataclasses.dataclass
class CVResult:
    cv: "object"       # torch.Tensor float64 [m] (device) or np.ndarray
    neff: "object"     # int64 [m]
    best: int
    h: np.ndarray

    @property
    def h_best(self) -> float:
        return float(self.h[self.best])


def shard_bounds(n: int, shard: int, nshards: int) -> tuple[int, int]:
    """Sorted-order rows [floor(r n / P), floor((r+1) n / P)) of shard r of P
    (the same rule kr_cv_shard_async applies on the device)."""
    if not (0 <= shard < nshards):
        raise ValueError("shard out of range")
    return (shard * n) // nshards, ((shard + 1) * n) // nshards


def allreduce_partial(partial, group=None) -> None:
    """The path's one exchange step: all-reduce(SUM) of the
    2m+2 partial vector [S | n_eff | n_bad_grid | n_nonfinite]; every entry
    is additive, so the reduced vector is the unsharded one."""
    import torch.distributed as dist

    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(partial, op=dist.ReduceOp.SUM, group=group)


def _nccl_group(group=None) -> bool:
    """True when torch.distributed is initialised with an NCCL group (whose
    collectives a CUDA graph can capture)."""
    import torch.distributed as dist

    return bool(dist.is_available() and dist.is_initialized() and dist.get_backend(group) == "nccl")


def finalize_partial(partial, n: int, m: int):
    """CV = S/n, n_eff and the arg-min from a reduced partial vector.  CUDA
    tensors are finalized on the device (kr_finalize_async), CPU tensors with
    the host entry point kr_finalize.  Returns (cv, neff, best)."""
    import torch

    if partial.is_cuda:
        cv = torch.empty(m, dtype=torch.float64, device=partial.device)
        neff = torch.empty(m, dtype=torch.int64, device=partial.device)
        bs = torch.empty(2, dtype=torch.int32, device=partial.device)
        krcv.kr_finalize_async(partial, n, m, cv, neff, bs)
        bs = bs.cpu()
        if int(bs[1]) != krcv.KR_OK:
            raise krcv.KrcvError(int(bs[1]), "device status")
        return cv, neff, int(bs[0])
    cv, neff, best = krcv.kr_finalize(partial.detach().numpy(), n, m)
    return torch.from_numpy(cv), torch.from_numpy(neff), best


def balanced_cuts(cost, n: int, world: int, align: int = 64) -> list[int]:
    """Row cut points [0, c_1, ..., c_{P-1}, n] of the sorted order that give
    every rank the same share of the measured cost.  cost[s]
    is the time of segment s of S equal segments [floor(s n / S),
    floor((s+1) n / S)); the cumulative cost is interpolated linearly inside
    a segment and every inner cut is rounded to a multiple of `align` rows
    (whole window-kernel tiles), kept non-decreasing within [0, n]."""
    cost = np.maximum(np.asarray(cost, np.float64), 0.0)
    S = cost.shape[0]
    if world <= 1 or S == 0 or not np.isfinite(cost).all() or cost.sum() <= 0.0:
        return [(r * n) // max(world, 1) for r in range(max(world, 1))] + [n]
    bounds = np.array([(s * n) // S for s in range(S + 1)], np.float64)
    cum = np.concatenate([[0.0], np.cumsum(cost)])
    cuts = [0]
    for r in range(1, world):
        target = cum[-1] * r / world
        s = int(np.searchsorted(cum, target, side="right")) - 1
        s = min(max(s, 0), S - 1)
        frac = 0.0 if cost[s] <= 0.0 else (target - cum[s]) / cost[s]
        row = bounds[s] + frac * (bounds[s + 1] - bounds[s])
        c = int(round(row / align)) * align
        cuts.append(min(max(c, cuts[-1]), n))
    cuts.append(n)
    return cuts


class GridSearch:
    """Reusable device plan for one (n, m, kernel) on one GPU / one rank.

    ``run(x, y)`` enqueues: sharded pipeline -> (all-reduce) -> device
    finalize, on the current stream; nothing synchronises until ``result()``.
    """

    def __init__(self, n: int, h, kernel="epanechnikov", device=None, rank: int = 0, world: int = 1,
                 group=None, algo="auto", estimator: str = "nw", graph: bool = False, balance: bool = False):
        import torch

        self.torch = torch
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        h_host = np.ascontiguousarray(h, dtype=np.float64)
        st = krcv.kr_validate_grid(h_host)
        if st != krcv.KR_OK:
            raise krcv.KrcvError(st, "grid")
        self.n, self.m = int(n), int(h_host.shape[0])
        self.kernel = krcv._kernel_id(kernel)
        self.algo = krcv._algo_id(algo)
        if estimator not in ("nw", "ll"):
            raise ValueError("estimator must be 'nw' (Nadaraya-Watson, Eq.(2)) or 'll' (local-linear, reading Q25)")
        self.estimator = estimator
        # graph=True: the enqueued pipeline is captured once per (x, y) pointer
        # pair as a CUDA graph and replayed -- one launch for the whole search
        # instead of one per stage.  With world > 1 (NCCL process group) the
        # captured step includes the shard's pipeline, the NCCL all-reduce of
        # the partial vector and the finalize; if the capture is refused (a
        # non-NCCL group, an NCCL/driver without graph support) the plan falls
        # back to eager enqueue and says so in self.graph_error.
        self.graph = bool(graph) and (int(world) == 1 or _nccl_group(group))
        self.graph_error = None
        self._g = None
        self._gkey = None
        self.rank, self.world, self.group = int(rank), int(world), group
        # balance=True (Nadaraya-Watson, world > 1): on the first run, rank 0
        # times the device path on 4 P equal row segments, cuts the sorted
        # rows at equal cumulative cost (balanced_cuts) and broadcasts the
        # cuts; every later run takes rows [cut_r, cut_{r+1}) through
        # kr_cv_rows_async.  Equal-row shards otherwise.
        self.balance = bool(balance) and self.world > 1 and estimator == "nw"
        self.rows = None
        self.h = h_host
        self.d_h = torch.as_tensor(h_host, device=self.device)
        self._ws_raw = krcv.workspace(self.n, self.m, self.device)
        self.ws = krcv.aligned(self._ws_raw)
        self.partial = torch.empty(krcv.partial_len(self.m), dtype=torch.float64, device=self.device)
        self.cv = torch.empty(self.m, dtype=torch.float64, device=self.device)
        self.neff = torch.empty(self.m, dtype=torch.int64, device=self.device)
        self.best_status = torch.empty(2, dtype=torch.int32, device=self.device)

    def run(self, d_x, d_y) -> None:
        if d_x.numel() != self.n or d_y.numel() != self.n:
            raise ValueError("x, y must have n elements")
        if self.graph:
            torch = self.torch
            key = (d_x.data_ptr(), d_y.data_ptr())
            if self._g is None or self._gkey != key:
                # eager first: one-time launch configuration queries (and, for
                # world > 1 with balance, the cost calibration and broadcast)
                self._enqueue(d_x, d_y)
                cur = torch.cuda.current_stream(self.device)
                side = torch.cuda.Stream(self.device)
                side.wait_stream(cur)
                g = torch.cuda.CUDAGraph()
                try:
                    with torch.cuda.graph(g, stream=side, capture_error_mode="thread_local"):
                        self._enqueue(d_x, d_y)
                except Exception as e:  # noqa: BLE001 -- capture refused: eager from now on
                    if self.world == 1:
                        raise
                    cur.wait_stream(side)
                    self.graph, self._g, self.graph_error = False, None, f"{type(e).__name__}: {e}"
                    self._enqueue(d_x, d_y)
                    return
                cur.wait_stream(side)
                self._g, self._gkey = g, key
            self._g.replay()
            return
        self._enqueue(d_x, d_y)

    def _enqueue(self, d_x, d_y) -> None:
        if self.estimator == "ll":
            if self.world == 1:
                krcv.kr_ll_cv_grid_async(d_x, d_y, self.d_h, self.kernel, self.cv, self.neff, self.best_status,
                                         self.ws)
                return
            krcv.kr_ll_shard_async(d_x, d_y, self.d_h, self.kernel, self.rank, self.world, self.partial, self.ws)
            allreduce_partial(self.partial, self.group)
            krcv.kr_finalize_async(self.partial, self.n, self.m, self.cv, self.neff, self.best_status)
            return
        if self.world == 1:  # whole search in one enqueue, finalize fused into the reduction
            krcv.kr_cv_grid_async(d_x, d_y, self.d_h, self.kernel, self.cv, self.neff, self.best_status, self.ws,
                                  algo=self.algo)
            return
        if self.balance:
            if self.rows is None:
                self.rows = self._balanced_rows(d_x, d_y)
            krcv.kr_cv_rows_async(d_x, d_y, self.d_h, self.kernel, self.rows[0], self.rows[1], self.partial,
                                  self.ws, algo=self.algo)
        else:
            krcv.kr_cv_shard_async(d_x, d_y, self.d_h, self.kernel, self.rank, self.world, self.partial, self.ws,
                                   algo=self.algo)
        allreduce_partial(self.partial, self.group)
        krcv.kr_finalize_async(self.partial, self.n, self.m, self.cv, self.neff, self.best_status)

    def _balanced_rows(self, d_x, d_y):
        """(lo, hi) of this rank from rank 0's cost measurement (broadcast)."""
        torch = self.torch
        import torch.distributed as dist

        cuts = torch.zeros(self.world + 1, dtype=torch.int64)
        if self.rank == 0:
            S = 4 * self.world
            cost = np.zeros(S)
            was_on = krcv.kr_profile_enabled()
            krcv.kr_profile_enable(True)
            try:
                for s in range(S):
                    lo, hi = (s * self.n) // S, ((s + 1) * self.n) // S
                    for _ in range(2):  # the second run is timed warm
                        krcv.kr_cv_rows_async(d_x, d_y, self.d_h, self.kernel, lo, hi, self.partial, self.ws,
                                              algo=self.algo)
                        cost[s] = krcv.kr_profile_read()[2]  # the window / sweep stage
            finally:
                krcv.kr_profile_enable(was_on)
            cuts = torch.tensor(balanced_cuts(cost, self.n, self.world), dtype=torch.int64)
        if dist.is_available() and dist.is_initialized():
            dev_cuts = cuts.to(self.device) if dist.get_backend(self.group) == "nccl" else cuts
            dist.broadcast(dev_cuts, src=dist.get_global_rank(self.group, 0) if self.group is not None else 0,
                           group=self.group)
            cuts = dev_cuts.cpu()
        c = [int(v) for v in cuts.tolist()]
        return c[self.rank], c[self.rank + 1]

    def result(self) -> CVResult:
        bs = self.best_status.cpu()
        st = int(bs[1])
        if st != krcv.KR_OK:
            raise krcv.KrcvError(st, "device status")
        # copies: the plan's buffers are overwritten by the next run() (or
        # graph replay), a result handed out must not change under the caller
        return CVResult(cv=self.cv.clone(), neff=self.neff.clone(), best=int(bs[0]), h=self.h)


def cv_grid(x, y, h=None, m: int | None = None, kernel="epanechnikov", device=None, distributed: bool = False,
            group=None, algo="auto", estimator: str = "nw", balance: bool = False) -> CVResult:
    """LOO-CV grid search.  x, y: numpy arrays or CUDA tensors; h: grid array,
    or None with m for the default grid (§IV P@16146).  With distributed=True
    every rank of the default (or given) process group must call it with the
    same inputs; the result is identical on every rank.  estimator: "nw"
    (Nadaraya-Watson, Eq.(2)) or "ll" (local-linear, reading Q25).
    balance: cost-balanced row cuts (GridSearch) -- a one-off calibration
    that pays off for plans run repeatedly, not for one call."""
    import torch

    if h is None:
        if m is None:
            raise ValueError("give h or m")
        xh = x.detach().cpu().numpy() if torch.is_tensor(x) else np.asarray(x, np.float64)
        h = krcv.kr_default_grid(xh, int(m))
    rank, world = 0, 1
    if distributed:
        import torch.distributed as dist

        rank, world = dist.get_rank(group), dist.get_world_size(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
    d_x = torch.as_tensor(x, dtype=torch.float64, device=dev).contiguous()
    d_y = torch.as_tensor(y, dtype=torch.float64, device=dev).contiguous()
    plan = GridSearch(d_x.numel(), h, kernel, dev, rank, world, group, algo, estimator, balance=balance)
    plan.run(d_x, d_y)
    return plan.result()


def cv_refine(x, y, h=None, m: int | None = None, kernel="epanechnikov", levels: int = 3, m_fine: int = 65,
              algo="auto"):
    """Coarse-to-fine search (§IV.A P@20112-20269; reading Q22) on the
    current CUDA device through kr_cv_refine: returns (h_best, cv_best), one
    entry per level.  h: level-0 grid, or None with m for the default grid."""
    xh = np.asarray(x, np.float64)
    if h is None:
        if m is None:
            raise ValueError("give h or m")
        h = krcv.kr_default_grid(xh, int(m))
    return krcv.kr_cv_refine(xh, np.asarray(y, np.float64), h, kernel, levels, m_fine, algo)
