"""Exact-rational brute force of Eq.(1)-(3) -- pin P1.

TEST INFRASTRUCTURE ONLY.

Straight from the definition (§III):
  Eq.(1) P@11484  CV(h) = n^-1 sum_i (Y_i - g_{-i}(X_i))^2 M(X_i)
  Eq.(2) P@11694  g_{-i}(X_i) = sum_{l!=i} Y_l K((X_i-X_l)/h) / sum_{l!=i} K(.)
         P@11802  M = 1 iff the denominator of (2) is non-zero
  Eq.(3) P@11971  K(u) = 0.75 (1 - u^2) I{|u| <= 1}
  fn.1   P@18521  uniform K = 1/2 I{|u|<=1}; triangular K = (1-|u|) I{|u|<1} (Q13)

Every value is a ``fractions.Fraction``; no sort, no running sum, no
decomposition.  Window membership follows reading Q1: decided in binary64 on
d = |x_l - x_i| (Python float subtraction is IEEE binary64), with '<' for
Epanechnikov/triangular and '<=' for uniform.  On the dyadic inputs the pins
use, binary64 subtraction is exact, so this equals the rational test.
M_i follows Q6 (at least one in-window neighbour), Q7 (M=0 rows add 0, divide
by n) and Q11 (smallest arg-min).
"""
from __future__ import annotations

from fractions import Fraction

UNIFORM, EPANECHNIKOV, TRIANGULAR = 0, 1, 2


def _K(u: Fraction, kernel: int) -> Fraction:
    if kernel == EPANECHNIKOV:
        return Fraction(3, 4) * (1 - u * u)
    if kernel == TRIANGULAR:
        return 1 - u
    return Fraction(1, 2)


def cv_exact(x, y, h, kernel: int):
    """Return (cv list of Fractions, neff list, best index)."""
    xs = [float(v) for v in x]
    ys = [Fraction(float(v)) for v in y]
    hs = [float(v) for v in h]
    n = len(xs)
    cvs, neffs = [], []
    for hb in hs:
        H = Fraction(hb)
        tot = Fraction(0)
        ne = 0
        for i in range(n):
            num = Fraction(0)
            den = Fraction(0)
            cnt = 0
            for l in range(n):
                if l == i:
                    continue
                d64 = abs(xs[l] - xs[i])
                inside = d64 <= hb if kernel == UNIFORM else d64 < hb
                if not inside:
                    continue
                u = abs(Fraction(xs[i]) - Fraction(xs[l])) / H
                w = _K(u, kernel)
                num += ys[l] * w
                den += w
                cnt += 1
            if cnt == 0:
                continue
            e = ys[i] - num / den
            tot += e * e
            ne += 1
        cvs.append(tot / n)
        neffs.append(ne)
    best = min(range(len(cvs)), key=lambda b: (cvs[b], b))
    return cvs, neffs, best


def cv_gauss_decimal(x, y, h, digits: int = 50):
    """Gaussian-kernel CV by the definition in decimal arithmetic with `digits`
    significant digits (exp by Decimal.exp): pin P1-G for the long-double
    oracle.  Eq.(2) with K(u) = exp(-u^2/2) (the normalising constant
    cancels); every l != i is in the window; no rescaling (the decimal exponent
    range makes underflow impossible here).  Returns (cv list of Decimal,
    best index)."""
    from decimal import Decimal, localcontext

    with localcontext() as ctx:
        ctx.prec = digits
        xs = [Decimal(float(v)) for v in x]
        ys = [Decimal(float(v)) for v in y]
        n = len(xs)
        cvs = []
        for hv in h:
            hh = Decimal(float(hv))
            two_h2 = 2 * hh * hh
            S = Decimal(0)
            for i in range(n):
                num = Decimal(0)
                den = Decimal(0)
                for l in range(n):
                    if l == i:
                        continue
                    d = xs[l] - xs[i]
                    w = (-(d * d) / two_h2).exp()
                    num += ys[l] * w
                    den += w
                e = ys[i] - num / den
                S += e * e
            cvs.append(S / n)
        best = min(range(len(cvs)), key=lambda b: (cvs[b], b))
        return cvs, best


def ll_cv_exact(x, y, h, kernel: int):
    """Local-linear LOO CV in exact rationals (pin for ``oracle.ll_cv``,
    reading Q25): per row and bandwidth, the 2x2 weighted normal equations
        [S0 S1; S1 S2] [a; beta] = [T0; T1],  S_k = sum w d^k, T_k = sum w y d^k,
    d = x_l - x_i, solved by Cramer's rule, a = (S2 T0 - S1 T1) / (S0 S2 - S1^2)
    -- the uncentred form, deliberately not the oracle's centred one.  A row is
    counted (M = 1) iff S0 S2 - S1^2 != 0.  Window membership as Q1 (binary64
    test on |d|).  Returns (cv list, neff list, best)."""
    xs = [float(v) for v in x]
    ys = [Fraction(float(v)) for v in y]
    n = len(xs)
    cvs, neffs = [], []
    for hb in (float(v) for v in h):
        H = Fraction(hb)
        tot, ne = Fraction(0), 0
        for i in range(n):
            S = [Fraction(0)] * 3
            T = [Fraction(0)] * 2
            for l in range(n):
                if l == i:
                    continue
                d64 = abs(xs[l] - xs[i])
                if not (d64 <= hb if kernel == UNIFORM else d64 < hb):
                    continue
                d = Fraction(xs[l]) - Fraction(xs[i])
                w = _K(abs(d) / H, kernel)
                S = [S[0] + w, S[1] + w * d, S[2] + w * d * d]
                T = [T[0] + w * ys[l], T[1] + w * ys[l] * d]
            det = S[0] * S[2] - S[1] * S[1]
            if det == 0:
                continue
            a = (S[2] * T[0] - S[1] * T[1]) / det
            tot += (ys[i] - a) ** 2
            ne += 1
        cvs.append(tot / n)
        neffs.append(ne)
    best = min(range(len(cvs)), key=lambda b: (cvs[b], b))
    return cvs, neffs, best


def _window(xs, i, l, hb, kernel):
    d64 = abs(xs[l] - xs[i])
    return d64 <= hb if kernel == UNIFORM else d64 < hb


def nw_jackknife_exact(x, y, hb: float, kernel: int):
    """Reading Q26 in exact rationals, by explicit deletion: for each point i,
    g_i = the Nadaraya-Watson estimate at x_i from the whole sample (i
    included), and for every j = 0..n-1 the estimate g_i^(-j) from the sample
    WITHOUT observation j, recomputed from scratch; the jackknife variance
    (n-1)/n sum_j (g_i^(-j) - mean_j g_i^(-j))^2.  No algebraic shortcut (the
    oracle's Delta_j form is what this checks).  Returns (est list, var list);
    var is None where some deletion empties the window."""
    xs = [float(v) for v in x]
    ys = [Fraction(float(v)) for v in y]
    n = len(xs)
    H = Fraction(float(hb))

    def estimate(i, skip):
        num = den = Fraction(0)
        for l in range(n):
            if l == skip or not _window(xs, i, l, float(hb), kernel):
                continue
            w = _K(abs(Fraction(xs[l]) - Fraction(xs[i])) / H, kernel)
            num += w * ys[l]
            den += w
        return None if den == 0 else num / den

    est, var = [], []
    for i in range(n):
        est.append(estimate(i, -1))
        dels = [estimate(i, j) for j in range(n)]
        if any(v is None for v in dels):
            var.append(None)
            continue
        mean = sum(dels) / n
        var.append(Fraction(n - 1, n) * sum((v - mean) ** 2 for v in dels))
    return est, var


def kde_jackknife_exact(x, hb: float, kernel: int):
    """Reading Q26 for the density, in exact rationals by explicit deletion:
    f_i = (1/(n h)) sum_j K(d_ij/h) with Q24's normalised kernels, the
    delete-one estimates f_i^(-j) = (1/((n-1) h)) sum_{l != j} K(d_il/h)
    recomputed from scratch, and their jackknife variance.  Returns
    (est list, var list)."""
    xs = [float(v) for v in x]
    n = len(xs)
    H = Fraction(float(hb))

    def k(i, l):
        if not _window(xs, i, l, float(hb), kernel):
            return Fraction(0)
        return _K(abs(Fraction(xs[l]) - Fraction(xs[i])) / H, kernel)

    est, var = [], []
    for i in range(n):
        kk = [k(i, l) for l in range(n)]
        tot = sum(kk)
        est.append(tot / (n * H))
        dels = [(tot - kk[j]) / ((n - 1) * H) for j in range(n)]
        mean = sum(dels) / n
        var.append(Fraction(n - 1, n) * sum((v - mean) ** 2 for v in dels))
    return est, var
