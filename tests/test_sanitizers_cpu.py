"""T7 on the CPU: the oracle's C code under AddressSanitizer
and UndefinedBehaviorSanitizer.  tests/sanitize/oracle_driver.c calls every
oracle entry point (all kernels, row subsets, n = 2, error paths) and is
compiled together with oracle/kr_oracle.c with -fsanitize=address,undefined
and -fno-sanitize-recover (any report aborts).  The device half of T7
(compute-sanitizer memcheck/racecheck/synccheck/initcheck on the CUDA path)
is tests/test_gpu_sanitizer.py.
"""
from __future__ import annotations

import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(shutil.which("gcc") is None, reason="gcc not available")
@pytest.mark.parametrize("real", ["ld", "d"])
def test_oracle_asan_ubsan(tmp_path, real):
    exe = str(tmp_path / f"oracle_san_{real}")
    cmd = ["gcc", "-O1", "-g", "-std=c11", "-fsanitize=address,undefined", "-fno-sanitize-recover=all",
           "-fno-omit-frame-pointer", "-fopenmp", "-ffp-contract=off", "-Wall",
           os.path.join(ROOT, "oracle", "kr_oracle.c"), os.path.join(ROOT, "tests", "sanitize", "oracle_driver.c"),
           "-o", exe, "-lm"]
    if real == "d":
        cmd.insert(1, "-DKRO_REAL=double")
    subprocess.run(cmd, check=True, capture_output=True, text=True)
    env = dict(os.environ, ASAN_OPTIONS="detect_leaks=1:abort_on_error=0", UBSAN_OPTIONS="print_stacktrace=1",
               OMP_NUM_THREADS="4")
    p = subprocess.run([exe], capture_output=True, text=True, env=env, timeout=300)
    assert p.returncode == 0, p.stdout[-2000:] + p.stderr[-4000:]
    assert "runtime error" not in p.stderr and "AddressSanitizer" not in p.stderr, p.stderr[-4000:]
    assert "ok" in p.stdout
