"""Offline replay of win_kernel's fast-path acceptance test (DESIGN.md §6.2,
"anchored records"): the fraction of (row, b) pairs that fail the test and
take the dd path, with the prefix records anchored at index 0 about the
median (round 1's records), or at J anchors (index-region centres, or spaced
evenly in x).  numpy float64 cumulative sums stand in for the rounded dd
records; rows are subsampled to ~20,000.  Measurement tool only: neither the
oracle nor the product imports it.

    python tools/anchor_replay.py C2 1 4 8 16
"""
import sys

import numpy as np

import workloads

KR = 32.0  # kFastTol / kFastSlack


def main():
    cfg = sys.argv[1]
    Js = [int(v) for v in sys.argv[2:]] or [1, 4, 8, 16]
    x, y, h, _ = workloads.make(cfg, seed=0)
    n = len(x)
    o_ = np.argsort(x, kind="stable")
    xs, ys = x[o_], y[o_]
    ymax = np.max(np.abs(ys))

    def pref(o, s0):
        u = xs - o
        T = np.stack([ys, u, u * u, ys * u, ys * u * u])
        P = np.zeros((5, n + 1))
        P[:, 1:] = np.cumsum(T, axis=1)
        return P - P[:, s0:s0 + 1]

    def fast(P, A, R, dl, hh, yr, c1):
        y_b, u_b, uu_b, yu_b, yuu_b = [P[i][R] for i in range(5)]
        y_a, u_a, uu_a, yu_a, yuu_a = [P[i][A] for i in range(5)]
        s1 = (uu_b - uu_a) - dl * (2 * (u_b - u_a) - c1 * dl)
        hk = hh * hh
        den = hk * (c1 - 1) - s1
        adl = np.abs(dl)
        ay = np.abs(y_b) + np.abs(y_a)
        E1 = np.abs(uu_b) + np.abs(uu_a) + 2 * adl * (np.abs(u_b) + np.abs(u_a)) + 2 * c1 * adl * (adl + hh)
        E2 = (np.abs(yuu_b) + np.abs(yuu_a) + 2 * adl * (np.abs(yu_b) + np.abs(yu_a)) + 2 * adl * adl * ay
              + 2 * c1 * ymax * adl * (adl + hh))
        E0 = ay + np.abs(yr)
        return (E1 <= KR * den) & (hk * E0 + E2 <= den * KR * ymax)

    rs = np.arange(0, n, max(1, n // 20000))

    def replay(anchors, by_x):
        anchors = np.unique(anchors)
        J = len(anchors)
        Ps = [pref(xs[a], a) for a in anchors]
        if by_x:
            ax = xs[anchors]
            pos = np.searchsorted(ax, xs[rs])
            lo, hi = np.clip(pos - 1, 0, J - 1), np.clip(pos, 0, J - 1)
            aj = np.where(np.abs(xs[rs] - ax[lo]) <= np.abs(xs[rs] - ax[hi]), lo, hi)
        else:
            aj = np.minimum((rs * J) // n, J - 1)
        tot = fail = 0
        for hh in h:
            xr, yr = xs[rs], ys[rs]
            R = np.searchsorted(xs, xr + hh, "left")
            A = np.searchsorted(xs, xr - hh, "right")
            c1 = (R - A).astype(float)
            ok = c1 > 1
            f = np.zeros(len(rs), bool)
            for j in range(J):
                sel = aj == j
                if sel.any():
                    f[sel] = fast(Ps[j], A[sel], R[sel], xr[sel] - xs[anchors[j]], hh, yr[sel], c1[sel])
            tot += ok.sum()
            fail += (ok & ~f).sum()
        return fail / tot

    base = pref(xs[n // 2], 0)
    tot = fail = 0
    for hh in h:
        xr, yr = xs[rs], ys[rs]
        R = np.searchsorted(xs, xr + hh, "left")
        A = np.searchsorted(xs, xr - hh, "right")
        c1 = (R - A).astype(float)
        ok = c1 > 1
        f = fast(base, A, R, xr - xs[n // 2], hh, yr, c1)
        tot += ok.sum()
        fail += (ok & ~f).sum()
    print(f"{cfg} round-1 records: dd fraction {fail / tot:.4f}")
    for J in Js:
        ai = (2 * np.arange(J) + 1) * n // (2 * J)
        ax = np.clip(np.searchsorted(xs, xs[0] + (np.arange(J) + 0.5) * (xs[-1] - xs[0]) / J), 0, n - 1)
        print(f"{cfg} J={J}: index-spaced anchors {replay(ai, False):.4f}, x-spaced {replay(ax, True):.4f}",
              flush=True)


if __name__ == "__main__":
    main()
