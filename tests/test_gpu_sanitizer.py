"""T7 on the GPU: compute-sanitizer memcheck, racecheck,
synccheck and initcheck over tests/sanitize/gpu_driver.py, which runs every
CUDA path of libkrcv.so once at small sizes (both sort paths, prefix build,
window kernel, sweep, histogram, Gaussian, KDE, local-linear, refinement,
reduction + fused finalize, the non-finite error path).  The
default window kernel and r01's (KRCV_WIN=r01) each get a racecheck run.
Any sanitizer report fails the test (--error-exitcode)."""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CS = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


def _run(tool: str, extra_env=None, args=()):
    if not os.path.exists(CS):
        pytest.skip("compute-sanitizer not found")
    env = dict(os.environ, **(extra_env or {}))
    env["PYTHONPATH"] = ROOT + os.pathsep + env.get("PYTHONPATH", "")
    cmd = [CS, "--tool", tool, "--error-exitcode", "99", *args, sys.executable,
           os.path.join(ROOT, "tests", "sanitize", "gpu_driver.py")]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    out = p.stdout + p.stderr
    if "compute-sanitizer is closed" in out:  # the pool's wrapper refuses every run (exit 86)
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    assert p.returncode == 0 and "gpu sanitizer driver: ok" in out, out[-6000:]
    assert "ERROR SUMMARY: 0 errors" in out or "RACECHECK SUMMARY: 0 hazards" in out, out[-6000:]


@pytest.mark.parametrize("tool", ["memcheck", "synccheck"])
def test_compute_sanitizer(tool):
    _run(tool, args=("--leak-check", "full") if tool == "memcheck" else ())


def test_compute_sanitizer_initcheck():
    _run("initcheck")


@pytest.mark.parametrize("win", ["default", "r01"])
def test_compute_sanitizer_racecheck(win):
    _run("racecheck", {} if win == "default" else {"KRCV_WIN": "r01", "KRCV_WIN_K": "2"})
