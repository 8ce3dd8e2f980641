"""Seeded synthetic workloads shared by the oracle side and the CUDA side.

This module holds input recipes ONLY -- random draws and the bandwidth-grid
spacing each workload is defined with. It contains none of the method's
arithmetic (no distances, windows, kernel weights, LOO estimates or CV sums),
so importing it from both `oracle/` and the product package does not couple
the two implementations.

Recipes:

* Generator: ``numpy.random.default_rng(seed)``; **x is drawn first, then the
  noise**. Arrays are float64 on the host.
* Paper DGP (PAPER.md P@16457-16803, §IV):  X ~ U(0,1),
  Y = 0.5 X + 10 X^2 + u,  u ~ U(0, 0.5).
* C1 (BASELINE.json configs[0]):  x ~ U(0, 2*pi), y = sin x + N(0, 0.5^2)
  (reading Q18: "N(0,0.25)" is the variance), default grid m=100, uniform kernel.
* C2-C4: paper DGP, default grid, Epanechnikov kernel.
* C5: x ~ LogNormal(0, 1), y = sin x + N(0, 0.5^2), 512 log-spaced bandwidths
  geomspace(1e-4 r, r), Epanechnikov kernel.

The default grid (PAPER.md P@16146-16375: max = range of X, min = range/k,
evenly spaced) is written here as the input recipe h_b = r * ((b+1)/m),
r = max(x) - min(x).  The library's ``kr_default_grid`` and the oracle's
``kro_default_grid`` implement the same rule independently; tests check all
three agree bit for bit.
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

UNIFORM = 0
EPANECHNIKOV = 1
TRIANGULAR = 2
GAUSSIAN = 3
KERNEL_NAMES = {UNIFORM: "uniform", EPANECHNIKOV: "epanechnikov", TRIANGULAR: "triangular",
                GAUSSIAN: "gaussian"}
KERNEL_IDS = {v: k for k, v in KERNEL_NAMES.items()}


@dataclasses.dataclass(frozen=True)
class Config:
    name: str
    n: int
    m: int
    kernel: int
    x_dist: str          # "paper" | "sin_uniform" | "lognormal"
    grid: str            # "default" | "log"
    note: str = ""


CONFIGS = {
    "C1": Config("C1", 1_000, 100, UNIFORM, "sin_uniform", "default",
                 "BASELINE configs[0]: oracle in seconds"),
    "C2": Config("C2", 20_000, 200, EPANECHNIKOV, "paper", "default",
                 "BASELINE configs[1]: paper's largest n, 1 GPU (bench headline)"),
    "C3": Config("C3", 100_000, 1_000, EPANECHNIKOV, "paper", "default",
                 "BASELINE configs[2]: 1 vs 8 GPUs"),
    "C4": Config("C4", 1_000_000, 1_000, EPANECHNIKOV, "paper", "default",
                 "BASELINE configs[3]: row-sharded across 8 GPUs"),
    "C5": Config("C5", 200_000, 512, EPANECHNIKOV, "lognormal", "log",
                 "BASELINE configs[4]: heavy tail, log grid"),
}


def draw_xy(kind: str, n: int, seed: int) -> tuple[np.ndarray, np.ndarray]:
    """Draw (x, y) for a workload family. x first, then the noise."""
    rng = np.random.default_rng(seed)
    if kind == "paper":
        x = rng.uniform(0.0, 1.0, n)
        u = rng.uniform(0.0, 0.5, n)
        y = 0.5 * x + 10.0 * x * x + u
    elif kind == "sin_uniform":
        x = rng.uniform(0.0, 2.0 * math.pi, n)
        e = rng.normal(0.0, 0.5, n)
        y = np.sin(x) + e
    elif kind == "lognormal":
        x = rng.lognormal(0.0, 1.0, n)
        e = rng.normal(0.0, 0.5, n)
        y = np.sin(x) + e
    else:
        raise ValueError(f"unknown x distribution {kind!r}")
    return np.ascontiguousarray(x, dtype=np.float64), np.ascontiguousarray(y, dtype=np.float64)


def grid_default(x: np.ndarray, m: int) -> np.ndarray:
    """Input recipe for the default grid: h_b = r * ((b+1)/m), r = max-min."""
    r = float(np.max(x)) - float(np.min(x))
    b1 = np.arange(1, m + 1, dtype=np.float64)
    return np.ascontiguousarray(r * (b1 / float(m)))


def grid_log(x: np.ndarray, m: int, lo_frac: float = 1e-4) -> np.ndarray:
    """Input recipe for C5: geomspace(lo_frac * r, r, m)."""
    r = float(np.max(x)) - float(np.min(x))
    h = np.geomspace(lo_frac * r, r, m)
    h[-1] = r
    return np.ascontiguousarray(np.maximum.accumulate(h))


def make(config: str | Config, seed: int = 0, n: int | None = None):
    """Return (x, y, h, kernel) for a named config (optionally resized to n rows)."""
    cfg = CONFIGS[config] if isinstance(config, str) else config
    nn = cfg.n if n is None else int(n)
    x, y = draw_xy(cfg.x_dist, nn, seed)
    h = grid_default(x, cfg.m) if cfg.grid == "default" else grid_log(x, cfg.m)
    return x, y, h, cfg.kernel


def random_dyadic(n: int, m: int, seed: int, dup: bool = True):
    """Small dyadic-rational inputs (exact in binary64, distances exact) for the
    exact brute-force pin: x, y are multiples of 1/8 in a small range; the grid
    contains values that coincide with pair distances (points exactly at h)."""
    rng = np.random.default_rng(seed)
    x = rng.integers(0, 24, n).astype(np.float64) / 8.0
    if dup and n >= 3:
        x[1] = x[0]
    y = rng.integers(-32, 33, n).astype(np.float64) / 8.0
    d = np.abs(x[:, None] - x[None, :])
    cand = np.unique(d[d > 0])
    picks = [] if cand.size == 0 else list(rng.choice(cand, size=min(m // 2, cand.size), replace=False))
    while len(picks) < m:
        picks.append(float(rng.integers(1, 32)) / 8.0)
    h = np.sort(np.array(picks[:m], dtype=np.float64))
    return np.ascontiguousarray(x), np.ascontiguousarray(y), np.ascontiguousarray(h)
