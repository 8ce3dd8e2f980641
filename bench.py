#!/usr/bin/env python
"""Benchmark: LOO-CV bandwidth grid search (Rohlfs & Zahran 2017) on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl ours|reference]

A "step" is one full grid search (every SURVEY.md §8(a) row: pack, sort,
sweep + LOO emit, reduce, [all-reduce], finalize/arg-min) over the config's
synthetic input, inputs resident in HBM.  Prints ONE JSON line (rank 0).

Metric (BASELINE.json): pair-bandwidth CV evaluations per second,
n (n-1) m / T_step, plus the wall time per full grid search (e2e).
For N > 1 (torchrun) rows are sharded across ranks with one NCCL all-reduce
of the 2m+2 partial vector; the job is fixed (strong scaling); time is the
max over ranks of CUDA-event time.

--impl reference times the CPU oracle (the paper's Program-3 algorithm,
oracle/kr_oracle.c) on the host cores on a bounded row sample of the same
workload (this tier's reference arm; there is no reference code).
"""
from __future__ import annotations

import argparse
import dataclasses
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads  # noqa: E402

METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
UNIT = "pair·bandwidth evals/s"
SM_COUNT = 148
FP64_LANES_PER_SM = 64          # FP64 FMA lanes per SM per clock
SM_MAX_MHZ_NOMINAL = 1965.0     # B200 clocks.max.sm (B200_PROFILING.md)
# Algorithmic FP64 flops (FMA = 2) per ordered pair and per (row, bandwidth)
# emit, per kernel.
FLOPS_PER_PAIR = {0: 2, 1: 6, 2: 5}
FLOPS_PER_EMIT = {0: 4, 1: 9, 2: 9}
# Window-prefix path: flops per (row, bandwidth) of its double-precision
# formula (prefix differences, shift to the row frame, estimate, error);
# DESIGN.md §6.2.
FLOPS_PER_WINDOW = {0: 6, 1: 25, 2: 30}
# FP64 operations of the two boundary lookups of one (row, bandwidth) in
# win_kernel (per side: x_r +- h, the bucket index FMA, four probes of
# subtract + compare): the search share of the work, for frac_incl_search.
SEARCH_FP64_PER_WINDOW = 20
# Small-message NCCL all-reduce latency over NVLink assumed by the P-GPU
# projection of other_configs (the 2m+2 fp64 partial vector, <= 16 KB); NOT
# measured here -- this environment has one GPU.
ALLREDUCE_US_ASSUMED = 20.0
# Dense Gaussian path: per (pair, bandwidth) x = t c (1), e^-x evaluated on
# the FP64 pipe (Cody-Waite 2 FMA + degree-12 Horner 12 FMA + rounding trick
# 2 + scale 1 = 31 flops), num FMA (2), den add (1).  DESIGN.md §6.5.
FLOPS_PER_PAIR_BW_DENSE = 35


def fp64_peak():
    """(TFLOP/s, note) of the FP64 roofline denominator: the DFMA throughput
    measured on a B200 of this pool by tools/fp64_peak.py (committed as
    profiles/fp64_peak.json with its clock record), else the derived nominal
    figure 148 x 64 x 2 x 1965 MHz."""
    try:
        with open(os.path.join(ROOT, "profiles", "fp64_peak.json")) as f:
            d = json.load(f)
        c = d.get("clocks", {})
        return float(d["dfma_tflops"]), (
            f"FP64 DFMA throughput measured by tools/fp64_peak.py on {d.get('gpu', 'B200')} "
            f"({d.get('when', '?')}, SM {c.get('sm_mhz')} of {c.get('sm_max_mhz')} MHz, reasons {c.get('reasons')}; "
            f"profiles/fp64_peak.json) -- of measured")
    except (OSError, ValueError, KeyError):
        return (SM_COUNT * FP64_LANES_PER_SM * 2 * SM_MAX_MHZ_NOMINAL * 1e6 / 1e12,
                "FP64: 148 SM x 64 FMA lanes x 2 flop x 1965 MHz (derived nominal; no measurement committed)")


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C2", choices=sorted(workloads.CONFIGS))
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-alt", action="store_true", help="skip timing the other algorithm (alt_algo)")
    ap.add_argument("--kde", action="store_true",
                    help="time the KDE least-squares CV (kr_kde_lscv_async, SURVEY §8(f) rank 3) on the config's x")
    ap.add_argument("--ll", action="store_true",
                    help="time the local-linear LOO CV (kr_ll_cv_grid_async, SURVEY §8(f) rank 4) on the config")
    ap.add_argument("--kernel", default=None, choices=["uniform", "epanechnikov", "triangular", "gaussian"],
                    help="override the config's kernel (e.g. the Gaussian dense path on C2's data)")
    ap.add_argument("--algo", default="auto", choices=["auto", "sweep", "prefix", "hist"],
                    help="KR_ALGO_* for every call (sets KRCV_ALGO before the library loads)")
    ap.add_argument("--no-extra", action="store_true",
                    help="skip the single-GPU C3/C4/C5 lines under other_configs (default run only)")
    ap.add_argument("--cpu-seconds", type=float, default=8.0,
                    help="target wall seconds of the bounded oracle sample")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def workload_desc(cfg, seed):
    kname = workloads.KERNEL_NAMES[cfg.kernel]
    return (f"{cfg.name}: n={cfg.n}, m={cfg.m} ({cfg.grid} grid), {kname} kernel, "
            f"x~{cfg.x_dist}, seed {seed}")


# --------------------------------------------------------------------- clocks
class ClockSampler:
    """Samples SM clock and throttle reasons through NVML during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, index: int):
        self.samples, self.reasons = [], 0
        self.max_mhz = None
        self._stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover - no NVML
            self.err = str(e)

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.reasons |= int(r) & ~0x1
            except Exception:
                pass
            time.sleep(0.002)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
            time.sleep(0.01)
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml_unavailable"]}
        names = [v for k, v in self.REASONS.items() if self.reasons & k]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples)}


def ncu_entry(config: str, algo: str):
    """The committed ncu capture's entry for this (config, algo)
    (profiles/ncu_traffic.json), else None."""
    try:
        with open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "ncu_traffic.json")) as f:
            return json.load(f).get(f"{config}/{algo}")
    except (OSError, ValueError):
        return None


def ncu_traffic(config: str, algo: str):
    """DRAM bytes per launch of the dominant kernel from the committed ncu
    capture for this (config, algo), else None."""
    e = ncu_entry(config, algo)
    return None if e is None else e.get("bytes")


def ncu_context(config: str, algo: str):
    """Pipe / issue / L1 counters of the same capture (what bounds frac)."""
    e = ncu_entry(config, algo)
    if e is None:
        return None
    return {k: v for k, v in e.items() if k not in ("bytes", "kernel")} or None


# --------------------------------------------------------------- cpu oracle
def oracle_sample(x, y, h, k, target_s: float):
    """Time the oracle (Program-3 algorithm) on a bounded row sample of the
    workload; returns (pair_bw_per_s, seconds, rows, threads)."""
    import oracle

    n, m = x.shape[0], h.shape[0]
    order = oracle.sorted_rows(x)
    threads = oracle.num_threads()
    rows = max(2 * threads, 16)
    evaluate = oracle.cv_direct if k == oracle.GAUSSIAN else oracle.cv_sorted  # no window to sweep (Q23)
    t0 = time.perf_counter()
    evaluate(x, y, h, k, rows=order[:rows])
    dt = time.perf_counter() - t0
    # size the sample from the measured per-row time; a small first probe
    # over-estimates it (thread start-up), so re-size until the sample takes
    # at least half the target (or covers every row)
    for _ in range(4):
        per_row = dt / rows
        rows = int(min(n, max(rows, 0.9 * target_s / max(per_row, 1e-9))))
        stride = max(1, n // rows)
        sample = order[::stride][:rows]  # spread over the sorted order
        t0 = time.perf_counter()
        evaluate(x, y, h, k, rows=sample)
        dt = time.perf_counter() - t0
        rows = int(sample.shape[0])
        if dt >= 0.5 * target_s or rows >= n:
            break
    return rows * (n - 1) * m / dt, dt, rows, threads


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# ------------------------------------------------------------ reference arm
def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    if world > 1 and os.environ.get("OMP_NUM_THREADS") == "1":
        # torchrun pins OMP_NUM_THREADS=1 per rank; rank 0 alone runs the
        # oracle here, on all of the host's cores (set before the oracle's
        # OpenMP runtime loads)
        os.environ["OMP_NUM_THREADS"] = str(len(os.sched_getaffinity(0)))
    cfg = workloads.CONFIGS[args.config]
    x, y, h, k = workloads.make(cfg, seed=args.seed)
    if args.kernel:
        k = workloads.KERNEL_IDS[args.kernel]
        cfg = dataclasses.replace(cfg, kernel=k)
    n, m = x.shape[0], h.shape[0]
    per_step_target = max(0.5, min(args.cpu_seconds, 120.0 / max(1, args.steps + args.warmup)))
    vals, secs, rows = [], [], 0
    threads = 1
    for s in range(args.warmup + args.steps):
        v, dt, rows, threads = oracle_sample(x, y, h, k, per_step_target)
        if s >= args.warmup:
            vals.append(v)
            secs.append(dt)
    value = statistics.median(vals)
    full_search_s = n * (n - 1) * m / value
    sample = (f"kro_cv_sorted (long double, per-row qsort + sweep) on {rows} of {n} rows "
              f"(strided over the x-sorted order), {threads} OpenMP threads; value extrapolated "
              f"to the full job; {cpu_model()}")
    out = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * full_search_s,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f80",
        "data": "synthetic",
        "config": {"workload": workload_desc(cfg, args.seed), "n": n, "m": m,
                   "kernel": workloads.KERNEL_NAMES[k], "seed": args.seed},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "wall_s_per_full_search_extrapolated": full_search_s,
    }
    print(json.dumps(out), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_ours(args):
    import torch

    rank, world, local = dist_env()
    if world != args.gpus:
        if world == 1 and args.gpus > 1:
            raise SystemExit("--gpus N>1 must be launched with torchrun (one rank per GPU)")
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device")
    # KRCV_BENCH_BACKEND=gloo (and more ranks than GPUs, ranks wrapping onto
    # the available devices) exercises the multi-rank code path on a one-GPU
    # box; the timed configuration is NCCL, one rank per GPU
    backend = os.environ.get("KRCV_BENCH_BACKEND", "nccl")
    local = local % torch.cuda.device_count() if backend != "nccl" else local
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    from paper_conf_ipps_rohlfsz17_b200 import krcv
    from paper_conf_ipps_rohlfsz17_b200.api import GridSearch

    cfg = workloads.CONFIGS[args.config]
    x, y, h, k = workloads.make(cfg, seed=args.seed)
    if args.kernel:
        k = workloads.KERNEL_IDS[args.kernel]
        cfg = dataclasses.replace(cfg, kernel=k)
    n, m = x.shape[0], h.shape[0]
    units = n * (n - 1) * m  # pair-bandwidth evaluations of one full grid search

    d_x = torch.as_tensor(x, device=dev)
    d_y = torch.as_tensor(y, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2
    stream = torch.cuda.current_stream(dev)
    rows_mine = ((rank + 1) * n) // world - (rank * n) // world
    main_wl = {"name": args.config, "x": x, "y": y, "h": h, "k": k, "n": n, "m": m, "d_x": d_x, "d_y": d_y, "units": units,
               "rows_mine": rows_mine}

    def barrier():
        if world > 1:
            torch.distributed.barrier()

    def timed(algo, wl=None, steps=None, warmup=None):
        """W warm-up + K device-timed grid searches with `algo`; L2 flushed
        between steps (outside the events); max over ranks.  wl: another
        workload (bench_extra_configs), default the config's."""
        wl = wl or main_wl
        nsteps = steps or args.steps
        nwarm = warmup or args.warmup
        x, y, h, k, n, m = wl["x"], wl["y"], wl["h"], wl["k"], wl["n"], wl["m"]
        cname = wl["name"]
        d_x, d_y, units, rows_mine = wl["d_x"], wl["d_y"], wl["units"], wl["rows_mine"]
        # single GPU: the whole search is replayed from a CUDA graph
        # (GridSearch(graph=True)).  Two plans: the headline steps replay a
        # graph WITHOUT the library's stage events; a second, profiled plan
        # (stage events captured as event-record nodes, profiling on before its
        # capture) gives the per-stage times, the dominant kernel's time for
        # the roofline and its share of a profiled step.
        def run_steps(plan, profiled):
            for _ in range(nwarm):
                plan.run(d_x, d_y)
            plan.result()
            torch.cuda.synchronize()
            starts = [torch.cuda.Event(enable_timing=True) for _ in range(nsteps)]
            ends = [torch.cuda.Event(enable_timing=True) for _ in range(nsteps)]
            st, launches = [], 0
            barrier()
            torch.cuda.synchronize()
            with ClockSampler(local) as clk:
                for s in range(nsteps):
                    flush.fill_(s & 0xFF)
                    starts[s].record(stream)
                    plan.run(d_x, d_y)
                    ends[s].record(stream)
                    if profiled:
                        st.append(krcv.kr_profile_read())  # syncs on this step's events
                    else:
                        ends[s].synchronize()
                    launches += krcv.kr_launch_count() + (1 if world > 1 else 0)  # + finalize (fused at N=1)
                torch.cuda.synchronize()
            barrier()
            # median step; the driver's clock brackets all K
            return statistics.median(starts[s].elapsed_time(ends[s]) for s in range(nsteps)), st, launches, clk

        krcv.kr_profile_enable(False)
        plan = GridSearch(n, h, k, device=dev, rank=rank, world=world, algo=algo, graph=True,
                          balance=(world > 1))
        step_ms, _, launches, clk = run_steps(plan, False)
        krcv.kr_profile_enable(True)
        pplan = GridSearch(n, h, k, device=dev, rank=rank, world=world, algo=algo, graph=True,
                          balance=(world > 1))
        prof_step_ms, st, _, _ = run_steps(pplan, True)
        krcv.kr_profile_enable(False)
        del pplan
        sort_ms, build_ms, main_ms, red_ms = ([v[i] for v in st] for i in range(4))
        used = {1: "sweep", 2: "prefix", 3: "dense", 4: "hist"}.get(krcv.kr_last_algo(), "?")
        main_med = statistics.median(main_ms)  # dominant kernel, median over the profiled steps
        if world > 1:
            t = torch.tensor([step_ms, main_med, prof_step_ms], dtype=torch.float64, device=dev)
            torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
            step_ms, main_med, prof_step_ms = float(t[0]), float(t[1]), float(t[2])
        res = plan.result()
        main_s = main_med * 1e-3
        peak, peak_note = fp64_peak()  # TFLOP/s
        if used == "dense":
            kname = "gauss_kernel (a3+a4, tiled all-pairs, Gaussian)"
            flops = rows_mine * (n - 1) * m * FLOPS_PER_PAIR_BW_DENSE
            basis = (f"{FLOPS_PER_PAIR_BW_DENSE} flops per (ordered pair, bandwidth) incl. the fp64 exp; "
                     "column truncation (weights < e^-64) not credited")
        elif used in ("sweep", "hist"):
            kname = ("sweep_kernel (a3+a4, per-pair running sums)" if used == "sweep" else
                     "hist_kernel (a3+a4, bucket-by-bandwidth smem histogram + warp scan)")
            flops = rows_mine * (n - 1) * FLOPS_PER_PAIR[k] + rows_mine * m * FLOPS_PER_EMIT[k]
            basis = (f"{FLOPS_PER_PAIR[k]} flops per ordered pair x rows x (n-1) + {FLOPS_PER_EMIT[k]} per "
                     "(row, bandwidth) emit")
        else:
            kname = "win_kernel (a3+a4, window-prefix with bucket-table boundary lookups)"
            flops = rows_mine * m * FLOPS_PER_WINDOW[k]
            basis = (f"{FLOPS_PER_WINDOW[k]} flops per (row, bandwidth): prefix differences, shift to the "
                     "row, LOO estimate, squared error (DESIGN.md §6.2); searches not counted (see "
                     "frac_incl_search)")
        achieved = flops / main_s / 1e12
        extra = {}
        if used == "prefix":
            fs = rows_mine * m * (FLOPS_PER_WINDOW[k] + SEARCH_FP64_PER_WINDOW)
            extra = {"flops_incl_search": fs, "frac_incl_search": fs / main_s / 1e12 / peak,
                     "search_basis": f"+{SEARCH_FP64_PER_WINDOW} FP64 ops per (row, bandwidth) for the two "
                                     "boundary lookups (x_r +- h, bucket index, four probes of subtract + "
                                     "compare per side; DESIGN.md §6.2)"}
        return {
            "algo": used, "value": units / (step_ms * 1e-3), "ms_per_step": step_ms,
            "stage_ms": {"pack_sort_gather": statistics.median(sort_ms), "prefix_build": statistics.median(build_ms),
                         "sweep": main_med, "reduce_finalize": statistics.median(red_ms)},
            "roofline": {"bound": "alu", "kernel": kname, "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": ncu_traffic(cname, used),
                         "ncu": ncu_context(cname, used),
                         "flops_per_launch": flops, "flops_basis": basis, **extra,
                         "peak_note": peak_note,
                         "kernel_ms": main_med,
                         "kernel_share_of_step": main_med / prof_step_ms,
                         "timing": "kernel_ms from stage CUDA events of a second, profiled run (events in its "
                                   "graph); value/ms_per_step from graph replays without stage events"},
            "ms_per_step_profiled": prof_step_ms,
            "timing_stat": "median over the K timed steps",
            "result": {"best": res.best, "h_best": float(h[res.best]), "cv_best": float(res.cv[res.best])},
            "clocks": clk.summary(), "gpu_launches": launches, "plan": plan,
            "launch": ("CUDA graph replay of the whole step" + (" incl. the NCCL all-reduce" if world > 1 else "")
                       if plan.graph else
                       (f"eager enqueue per step (graph capture refused: {plan.graph_error})" if plan.graph_error
                        else "eager enqueue per step (non-NCCL process group: collectives not capturable)")),
        }

    main = timed(args.algo)
    plan = main.pop("plan")
    main_launch = main.pop("launch")

    # ---- end-to-end through the public API, host buffers, H2D/D2H inside
    e2e = e2e_measure(args, x, y, h, k, n, m, units, dev, rank, world, plan)

    out = {
        "metric": METRIC, "value": main["value"], "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": main["ms_per_step"], "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_desc(cfg, args.seed), "n": n, "m": m,
                   "kernel": workloads.KERNEL_NAMES[k], "seed": args.seed,
                   "parallelism": f"row-shard x{world}" + (
                       " (cost-balanced cuts from rank 0's calibration in the first warm-up step)"
                       f" + {os.environ.get('KRCV_BENCH_BACKEND', 'nccl')} all_reduce(2m+2 fp64)" if world > 1 else ""),
                   "l2": "flushed between timed steps (256 MiB write, outside the events)",
                   "launch": main_launch},
        "algo": main["algo"],
        "roofline": main["roofline"],
        "stage_ms": main["stage_ms"],
        "ms_per_step_profiled": main["ms_per_step_profiled"],
        "result": main["result"],
        "e2e": e2e,
        "clocks": main["clocks"],
        "gpu_launches": main["gpu_launches"],
        "wall_time_per_grid_search_ms": e2e.get("ms_per_search"),
    }
    if not args.no_alt and main["algo"] != "dense":
        other = "sweep" if main["algo"] == "prefix" else "prefix"
        alt = timed(other)
        alt.pop("plan")
        alt.pop("launch")
        out["alt_algo"] = {key: alt[key] for key in ("algo", "value", "ms_per_step", "stage_ms", "roofline",
                                                      "result", "clocks")}
    if world == 1 and args.config == "C2" and not args.no_extra:
        out["other_configs"] = bench_extra_configs(args, timed, dev, krcv, torch)
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, dt, rows, threads = oracle_sample(x, y, h, k, args.cpu_seconds)
        out["cpu_baseline"] = {
            "value": v, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": (f"{'kro_cv_direct' if k == 3 else 'kro_cv_sorted'} on {rows} of {n} rows "
                       "(strided over the x-sorted order), "
                       f"{dt:.1f} s, {threads} OpenMP threads, {cpu_model()}; extrapolated to the full job")}
    if world > 1:
        torch.distributed.barrier()
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()
    return 0


def bench_extra_configs(args, timed, dev, krcv, torch):
    """The other BASELINE.json configurations on this one GPU (C3, C4, C5:
    configs[2..4]) in the same launch configuration as the headline, each with
    its stage times and roofline, plus the row-shard balance of the window
    stage at P = 2, 4, 8 (the P sorted-row shards timed one after another on
    this GPU through kr_cv_rows_async; equal rows and cost-balanced cuts) and
    the projected P-GPU time
        T(P) = pack/sort + prefix/table build (replicated on every rank; of
               the anchored copies only those of the rank's rows, the
               slowest shard's build timed) + window * (max shard / mean
               shard) / P + reduce
               + ALLREDUCE_US_ASSUMED
    and efficiency T(1) / (P T(P)).  A projection from single-GPU stage times,
    not a multi-GPU measurement (this environment has one GPU)."""
    res = {}
    for name in ("C3", "C4", "C5"):
        cfg = workloads.CONFIGS[name]
        x, y, h, k = workloads.make(cfg, seed=args.seed)
        n, m = x.shape[0], h.shape[0]
        wl = {"name": name, "x": x, "y": y, "h": h, "k": k, "n": n, "m": m, "d_x": torch.as_tensor(x, device=dev),
              "d_y": torch.as_tensor(y, device=dev), "units": n * (n - 1) * m, "rows_mine": n}
        r = timed("auto", wl, steps=5 if name == "C4" else 10, warmup=3)
        r.pop("plan")
        r.pop("launch")
        # window-stage balance of P row shards: equal rows, and the
        # cost-balanced cuts bench.py uses at N > 1 (api.balanced_cuts from 4P
        # calibration segments)
        from paper_conf_ipps_rohlfsz17_b200 import api as _api

        d_h = torch.as_tensor(h, device=dev)
        ws = krcv.aligned(krcv.workspace(n, m, dev))
        part = torch.zeros(krcv.partial_len(m), dtype=torch.float64, device=dev)
        krcv.kr_profile_enable(True)

        def stages_ms(lo, hi):
            for _ in range(2):  # the second run is timed (warm)
                krcv.kr_cv_rows_async(wl["d_x"], wl["d_y"], d_h, k, lo, hi, part, ws)
                t = krcv.kr_profile_read()
            return t

        def window_ms(lo, hi):
            return stages_ms(lo, hi)[2]

        imb_eq, imb_bal, cuts_bal, build_bal = {}, {}, {}, {}
        shard8 = []
        for P in (2, 4, 8):
            eq = [window_ms((s * n) // P, ((s + 1) * n) // P) for s in range(P)]
            if P == 8:
                shard8 = eq
            imb_eq[P] = max(eq) / (sum(eq) / P)
            calib = [window_ms((s * n) // (4 * P), ((s + 1) * n) // (4 * P)) for s in range(4 * P)]
            cuts = _api.balanced_cuts(calib, n, P)
            tb = [stages_ms(cuts[s], cuts[s + 1]) for s in range(P)]
            bal = [t[2] for t in tb]
            imb_bal[P] = max(bal) / (sum(bal) / P)
            # a rank's O(n) build: the prefix, the table and only the anchored
            # copies its rows use -- the slowest shard's
            build_bal[P] = max(t[1] for t in tb)
            cuts_bal[P] = cuts
        krcv.kr_profile_enable(False)
        del ws
        st = r["stage_ms"]
        t1 = r["ms_per_step"]
        fixed = st["reduce_finalize"] + ALLREDUCE_US_ASSUMED * 1e-3
        repl = st["pack_sort_gather"] + st["prefix_build"]
        proj, proj_eq, bound = {}, {}, {}
        for P in (2, 4, 8):
            repl_p = st["pack_sort_gather"] + build_bal[P]
            tp = repl_p + st["sweep"] * imb_bal[P] / P + fixed
            proj[str(P)] = {"ms": tp, "efficiency": t1 / (P * tp), "imbalance": imb_bal[P],
                            "replicated_ms": repl_p}
            tq = repl + st["sweep"] * imb_eq[P] / P + fixed
            proj_eq[str(P)] = {"ms": tq, "efficiency": t1 / (P * tq), "imbalance": imb_eq[P]}
            tb = st["sweep"] * imb_bal[P] / P + fixed
            bound[str(P)] = t1 / (P * tb)
        res[name] = {"workload": workload_desc(cfg, args.seed), "value": r["value"], "unit": UNIT,
                     "ms_per_step": t1, "stage_ms": st, "roofline": r["roofline"], "result": r["result"],
                     "clocks": r["clocks"], "gpu_launches": r["gpu_launches"],
                     "shard8_window_ms": shard8, "shard8_imbalance": imb_eq[8],
                     "projected_scaling": proj,
                     "projected_scaling_equal_rows": proj_eq,
                     "efficiency_bound_no_replicated_stage": bound,
                     "balanced_cuts": {str(P): c for P, c in cuts_bal.items()},
                     "projection_note": ("T(P) = replicated sort + the slowest balanced shard's prefix/table/anchor "
                                         "build (a rank builds only its rows' anchored copies; equal rows: the "
                                         "whole single-GPU build) + window x imbalance(P) / P "
                                         f"+ reduce + {ALLREDUCE_US_ASSUMED} us assumed all-reduce; imbalance = "
                                         "max/mean window time of the P shards, timed one after another on this "
                                         "GPU (cost-balanced cuts, as bench.py runs N > 1; equal rows in "
                                         "projected_scaling_equal_rows); efficiency_bound_no_replicated_stage "
                                         "drops the sort + build (the Amdahl bound of a fully distributed O(n) "
                                         "stage); one-GPU stage times, not a multi-GPU measurement")}
    return res


def e2e_measure(args, x, y, h, k, n, m, units, dev, rank, world, plan):
    """Same metric through the public API from pinned host buffers, per step:
    H2D of x, y (and h), the grid search, D2H of the CV curve and best."""
    import ctypes

    import torch

    from paper_conf_ipps_rohlfsz17_b200 import krcv

    hx = torch.from_numpy(x).pin_memory()
    hy = torch.from_numpy(y).pin_memory()
    hh = torch.from_numpy(h).pin_memory()
    hcv = torch.empty(m, dtype=torch.float64).pin_memory()
    times = []
    if world == 1:
        best = ctypes.c_int32(-1)
        for s in range(args.warmup + args.steps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st = krcv.kr_cv_grid_ptr(hx.data_ptr(), hy.data_ptr(), n, hh.data_ptr(), m, k, hcv.data_ptr(),
                                     ctypes.byref(best))
            t1 = time.perf_counter()
            if st != 0:
                raise krcv.KrcvError(st, "kr_cv_grid")
            if s >= args.warmup:
                times.append(t1 - t0)
        api = "kr_cv_grid (C-ABI, host pointers, synchronous)"
        d2h = 16 * m + 8  # one result block: [best, status] | cv[m] | neff[m]
    else:
        d_x = torch.empty(n, dtype=torch.float64, device=dev)
        d_y = torch.empty(n, dtype=torch.float64, device=dev)
        for s in range(args.warmup + args.steps):
            torch.distributed.barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            d_x.copy_(hx, non_blocking=True)
            d_y.copy_(hy, non_blocking=True)
            plan.run(d_x, d_y)
            hcv.copy_(plan.cv, non_blocking=True)
            bs = plan.best_status.cpu()
            t1 = time.perf_counter()
            if int(bs[1]) != 0:
                raise krcv.KrcvError(int(bs[1]), "device status")
            if s >= args.warmup:
                times.append(t1 - t0)
        t = torch.tensor([sum(times)], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        times = [float(t[0]) / len(times)] * len(times)
        api = "GridSearch.run (row-sharded, NCCL all-reduce) with pinned H2D/D2H per step"
        d2h = 8 * m + 8
    med = statistics.median(times)
    return {"value": units / med, "unit": UNIT, "h2d_bytes_per_step": 16 * n + 8 * m,
            "d2h_bytes_per_step": d2h, "ms_per_search": 1e3 * med, "api": api,
            "timing": "host wall clock around the synchronous call, median over the K steps"}


def run_kde(args):
    """KDE LSCV (reading Q24) on the config's x: device-timed whole searches,
    pair-bandwidth evaluations n (n-1) m per second; one JSON line."""
    import torch

    from paper_conf_ipps_rohlfsz17_b200 import krcv

    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    cfg = workloads.CONFIGS[args.config]
    x, _, h, k = workloads.make(cfg, seed=args.seed)
    if args.kernel:
        k = workloads.KERNEL_IDS[args.kernel]
    n, m = x.shape[0], h.shape[0]
    d_x = torch.as_tensor(x, device=dev)
    d_h = torch.as_tensor(h, device=dev)
    ws = krcv.aligned(krcv.workspace(n, m, dev))
    out = torch.empty(m, dtype=torch.float64, device=dev)
    bs = torch.empty(2, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream(dev)
    lib = krcv._lib()

    def run():
        st = lib.kr_kde_lscv_async(d_x.data_ptr(), n, d_h.data_ptr(), m, k, out.data_ptr(), bs.data_ptr(),
                                   ws.data_ptr(), ws.numel(), __import__("ctypes").c_void_p(stream.cuda_stream))
        if st:
            raise krcv.KrcvError(st, "kr_kde_lscv_async")

    for _ in range(args.warmup):
        run()
    torch.cuda.synchronize()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    krcv.kr_profile_enable(True)
    tot, win = 0.0, 0.0
    with ClockSampler(0) as clk:
        for s_ in range(args.steps):
            flush.fill_(s_ & 0xFF)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            run()
            b.record(stream)
            stg = krcv.kr_profile_read()
            win += stg[2]
            tot += a.elapsed_time(b)
    krcv.kr_profile_enable(False)
    best = int(bs[0])
    units = n * (n - 1) * m
    print(json.dumps({
        "metric": "KDE LSCV pair-bandwidth evals/s (SURVEY 8(f) rank 3)", "value": units * args.steps / (tot * 1e-3),
        "unit": UNIT, "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot / args.steps,
        "higher_is_better": True, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name} x, kde lscv, {workloads.KERNEL_NAMES[k]}", "n": n, "m": m},
        "kde_window_kernel_ms": win / args.steps, "result": {"best": best, "h_best": float(h[best]),
                                                              "lscv_best": float(out[best])},
        "clocks": clk.summary()}), flush=True)
    return 0


# Local-linear algorithmic work per (row, bandwidth), Epanechnikov, in the
# double formula: 9 prefix differences, binomial shifts of
# D1..D4 (10 multiply-adds) and Y0..Y3 (6), S0..S2, T0, T1 (5 FMA), det and
# num (2 x 3), g (1), e^2 and its sum (3): 61 flops.  Uniform: 5 differences,
# shifts D1, D2, Y1 (4 multiply-adds), det/num (6), g, e^2, sum (4): 23.
LL_FLOPS = {0: 23, 1: 61, 2: 2 * 61}


def run_ll(args):
    """Local-linear LOO CV (reading Q25) on the config: device-timed whole
    searches (kr_ll_cv_grid_async), pair-bandwidth evaluations n (n-1) m per
    second, the window kernel's FP64 roofline fraction; one JSON line."""
    import ctypes

    import torch

    from paper_conf_ipps_rohlfsz17_b200 import krcv

    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    cfg = workloads.CONFIGS[args.config]
    x, y, h, k = workloads.make(cfg, seed=args.seed)
    if args.kernel:
        k = workloads.KERNEL_IDS[args.kernel]
    n, m = x.shape[0], h.shape[0]
    d_x, d_y, d_h = (torch.as_tensor(a, device=dev) for a in (x, y, h))
    ws = krcv.aligned(krcv.workspace(n, m, dev))
    cv = torch.empty(m, dtype=torch.float64, device=dev)
    bs = torch.empty(2, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream(dev)
    lib = krcv._lib()

    def run():
        st = lib.kr_ll_cv_grid_async(d_x.data_ptr(), d_y.data_ptr(), n, d_h.data_ptr(), m, k, cv.data_ptr(), None,
                                     bs.data_ptr(), ws.data_ptr(), ws.numel(), ctypes.c_void_p(stream.cuda_stream))
        if st:
            raise krcv.KrcvError(st, "kr_ll_cv_grid_async")

    for _ in range(args.warmup):
        run()
    torch.cuda.synchronize()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    krcv.kr_profile_enable(True)
    tot, win = 0.0, 0.0
    stages = [0.0] * 4
    with ClockSampler(0) as clk:
        for s_ in range(args.steps):
            flush.fill_(s_ & 0xFF)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            run()
            b.record(stream)
            stg = krcv.kr_profile_read()
            stages = [u + v for u, v in zip(stages, stg)]
            tot += a.elapsed_time(b)
    krcv.kr_profile_enable(False)
    best = int(bs[0])
    units = n * (n - 1) * m
    kms = stages[2] / args.steps
    flops = LL_FLOPS.get(k, 61) * n * m
    peak, _ = fp64_peak()  # TFLOP/s, as run_ours
    ach = flops / (kms * 1e-3) / 1e12
    print(json.dumps({
        "metric": "local-linear LOO-CV pair-bandwidth evals/s (SURVEY 8(f) rank 4)",
        "value": units * args.steps / (tot * 1e-3), "unit": UNIT, "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": tot / args.steps, "higher_is_better": True, "dtype": "f64",
        "data": "synthetic",
        "config": {"workload": f"{cfg.name}, local-linear, {workloads.KERNEL_NAMES[k]}", "n": n, "m": m,
                   "l2": "flushed between timed steps (256 MiB write, outside the events)"},
        "roofline": {"bound": "alu", "kernel": "ll_window_kernel", "achieved": ach, "peak": peak, "unit": "TFLOP/s",
                     "frac": ach / peak, "traffic": None, "flops_per_launch": flops,
                     "flops_basis": f"{LL_FLOPS.get(k, 61)} flops per (row, bandwidth) in the double formula "
                                    "(DESIGN.md 6.7); dd arithmetic and searches not counted",
                     "kernel_ms": kms, "kernel_share_of_step": kms / (tot / args.steps)},
        "stage_ms": {"pack_sort_gather": stages[0] / args.steps, "prefix_build": stages[1] / args.steps,
                     "window": kms, "reduce_finalize": stages[3] / args.steps},
        "result": {"best": best, "h_best": float(h[best]), "cv_best": float(cv[best])},
        "clocks": clk.summary()}), flush=True)
    return 0


def main():
    args = parse()
    if args.kde:
        return run_kde(args)
    if args.ll:
        return run_ll(args)
    if args.algo != "auto":
        os.environ["KRCV_ALGO"] = args.algo
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
