"""The C-ABI used from plain C (examples/krcv_example.c): compiled with gcc
against include/krcv.h and linked to libkrcv.so, without Python or PyTorch in
the process.  CPU tier: the host-only entry points (version, default grid,
grid validation, argument errors); GPU tier: a whole search from plain C --
the full CV curve and n_eff (kr_cv_grid_ex) against the oracle element by
element, the optimum, and the leave-one-out confidence intervals at it
(kr_cv_ci, reading Q26) for every observation."""
from __future__ import annotations

import os
import re
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIBDIR = os.path.join(ROOT, "paper_conf_ipps_rohlfsz17_b200")


def _build(tmp_path):
    if shutil.which("gcc") is None:
        pytest.skip("gcc not available")
    exe = str(tmp_path / "krcv_example")
    subprocess.run(["gcc", "-O2", "-std=c11", "-Wall", "-I", os.path.join(ROOT, "include"),
                    os.path.join(ROOT, "examples", "krcv_example.c"), "-L", LIBDIR, "-lkrcv",
                    f"-Wl,-rpath,{LIBDIR}", "-o", exe], check=True, capture_output=True, text=True)
    return exe


def test_c_consumer_host_only(tmp_path):
    p = subprocess.run([_build(tmp_path), "--host-only"], capture_output=True, text=True, timeout=120)
    assert p.returncode == 0, p.stdout + p.stderr
    assert "sm_100a" in p.stdout and "host-only ABI checks: ok" in p.stdout


@pytest.mark.gpu
def test_c_consumer_full_search(tmp_path):
    import numpy as np

    import oracle
    p = subprocess.run([_build(tmp_path), "3000", "40", "--dump"], capture_output=True, text=True, timeout=300)
    assert p.returncode == 0, p.stdout + p.stderr
    mt = re.search(r"best b = (\d+), h = (\S+), CV = (\S+)", p.stdout)
    assert mt, p.stdout
    # the same xorshift inputs, regenerated here for the oracle
    s = 0x9E3779B97F4A7C15
    mask = (1 << 64) - 1

    def urand():
        nonlocal s
        s ^= (s << 13) & mask
        s ^= s >> 7
        s ^= (s << 17) & mask
        return (s >> 11) * 2.0 ** -53

    n, m = 3000, 40
    x = np.empty(n)
    y = np.empty(n)
    for i in range(n):
        x[i] = urand()
        y[i] = 0.5 * x[i] + 10.0 * x[i] * x[i] + 0.5 * urand()
    h = oracle.default_grid(x, m)
    ref = oracle.cv_sorted(x, y, h, oracle.EPANECHNIKOV)
    assert int(mt.group(1)) == ref.best
    assert abs(float(mt.group(3)) - ref.cv[ref.best]) <= 1e-9 * ref.cv[ref.best]
    from tests.helpers import cv_rel_err

    curve = [ln.split() for ln in p.stdout.splitlines() if ln.startswith("curve ")]
    assert [int(c[1]) for c in curve] == list(range(m))
    cv = np.array([float(c[2]) for c in curve])
    neff = np.array([int(c[3]) for c in curve])
    assert cv_rel_err(cv, ref.cv) <= 1e-10
    assert np.array_equal(neff, ref.neff)
    ci = [ln.split() for ln in p.stdout.splitlines() if ln.startswith("ci ")]
    assert [int(c[1]) for c in ci] == list(range(n))
    est = np.array([float(c[2]) for c in ci])
    se = np.array([float(c[3]) for c in ci])
    jk = oracle.nw_jackknife(x, y, float(h[ref.best]), oracle.EPANECHNIKOV)
    assert np.max(np.abs(est - jk.est) / np.abs(jk.est)) <= 1e-10
    ok = ~np.isnan(jk.se)
    assert np.array_equal(np.isnan(se), ~ok)
    assert np.max(np.abs(se[ok] - jk.se[ok]) / jk.se[ok]) <= 1e-10
