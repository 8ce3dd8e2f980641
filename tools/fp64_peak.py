#!/usr/bin/env python
"""Measured FP64 peak of this GPU: the roofline denominator bench.py divides by.

    python tools/fp64_peak.py [--out profiles/fp64_peak.json]

Times tools/libfp64peak.so (DFMA / DADD throughput kernels, tools/fp64_peak.cu)
with CUDA events while bench.py's NVML sampler records the SM clock and the
throttle reasons, and writes one JSON object: DFMA TFLOP/s (FMA = 2 flops),
DADD Gop/s, the clocks seen, and the derived nominal figure for comparison
(148 SM x 64 FP64 lanes x 2 x clocks.max.sm).
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

LIB = os.path.join(ROOT, "tools", "libfp64peak.so")


def measure(iters: int = 20000, reps: int = 5) -> dict:
    import torch

    from bench import ClockSampler, SM_COUNT, FP64_LANES_PER_SM

    lib = ctypes.CDLL(LIB)
    lib.fp64_peak_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                  ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]
    torch.cuda.set_device(0)
    st = torch.cuda.current_stream().cuda_stream
    res = {}
    with ClockSampler(0) as clk:
        for name, fma in (("dfma", 1), ("dadd", 0)):
            ms, fl = ctypes.c_double(), ctypes.c_double()
            rc = lib.fp64_peak_run(fma, iters, reps, ctypes.c_void_p(st), ctypes.byref(ms), ctypes.byref(fl))
            if rc:
                raise RuntimeError(f"fp64_peak_run({name}) -> cudaError {rc}")
            res[name] = {"ms": ms.value, "flops": fl.value, "tflops": fl.value / (ms.value * 1e-3) / 1e12}
    c = clk.summary()
    max_mhz = c.get("sm_max_mhz") or 1965.0
    nominal = SM_COUNT * FP64_LANES_PER_SM * 2 * max_mhz * 1e6 / 1e12
    return {
        "what": "FP64 throughput, tools/fp64_peak.cu: 148x8 CTAs x 256 threads, 8 independent DFMA (DADD) chains "
                "per thread, best of %d launches, CUDA events" % reps,
        "dfma_tflops": res["dfma"]["tflops"],
        "dadd_gops": res["dadd"]["tflops"] * 1e3,
        "dfma_ms": res["dfma"]["ms"],
        "nominal_tflops_at_max_clock": nominal,
        "dfma_frac_of_nominal": res["dfma"]["tflops"] / nominal,
        "clocks": c,
        "gpu": torch.cuda.get_device_name(0),
        "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()),
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    r = measure()
    line = json.dumps(r)
    print(line)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main()
