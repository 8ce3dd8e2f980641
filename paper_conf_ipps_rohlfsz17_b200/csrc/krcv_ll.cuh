// krcv_ll.cuh -- local-linear leave-one-out CV on the window-prefix path
// (§IV P@15728 "The Nadaraya-Watson [19],
// [27] local constant estimator is used rather than a local linear
// regression"; reading Q25).
//
// For sorted row r and bandwidth h the LOO local-linear estimate is the
// intercept of the kernel-weighted least-squares line through the window
// W_r(h) \ {r} (the same window as Eq.(2), reading Q1):
//     g = (S2 T0 - S1 T1) / (S0 S2 - S1^2),
//     S_k = sum w d^k,  T_k = sum w y d^k,  d = x_l - x_r,
// with the weights of Eq.(3) / footnote 1 up to a constant factor (it
// cancels): uniform w = 1, Epanechnikov w = h^2 - d^2, triangular
// w = h - |d|.  So S_k and T_k are polynomials in the window's power sums
//     D_k = sum d^k  (k <= 4),   Y_k = sum y d^k  (k <= 3),
// which the prefix moments u^k and y u^k (u = x - o, double-double,
// krcv_prefix.cuh) give in O(1) per (row, bandwidth) by the binomial shift
//     D_k = sum_i C(k,i) U_i (-delta)^(k-i),  delta = x_r - o,
// evaluated in dd.  The triangular weight needs |d|: its sums are split at
// the row (right d > 0, left d < 0).
//
// Row r's own terms vanish (d = 0) except in the count and in Y_0, which
// subtract them.  M_r = [the window holds >= 2 distinct x] (reading Q25) is
// an exact test on the sorted x: its first and last element differ.
//
// Accuracy: the prefix differences and the shift carry an absolute error
// bounded by kappa * mag_k (kappa = (n + 64) 2^-104 covers the prefix
// build's accumulated dd rounding, mag_k = the binomial combination of the
// prefix magnitudes); S, T, det = S0 S2 - S1^2 and num = S2 T0 - S1 T1
// stay in dd (det cancels badly when the window sits far to one side of the
// row: tail rows at large h), and the propagated bound covers g.  If the bound is not below 2^-44 max|y| (or the window is small,
// c <= kLLDirect, where the direct loop is cheaper anyway) g is computed
// directly over the window in the centred two-pass form.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "krcv.h"
#include "krcv_dd.cuh"
#include "krcv_prefix.cuh"

namespace krcv {

constexpr int kLLDirect = 16;  // windows up to this many points: direct two-pass

// w(d) up to the constant factor of the kernel (cancels in g)
template <int KERN>
__device__ __forceinline__ double ll_weight(double ad, double h)
{
    if (KERN == KR_UNIFORM) return 1.0;
    if (KERN == KR_EPANECHNIKOV) return (h - ad) * (h + ad);
    return h - ad;
}

// g over [A, R) \ {r} directly: weighted means, then the centred slope.
template <int KERN>
__device__ double ll_direct(const double2 *__restrict__ xy, int A, int R, int r, double xr, double h)
{
    double s0 = 0.0, sd = 0.0, sy = 0.0;
    for (int q = A; q < R; q++) {
        if (q == r) continue;
        const double2 v = xy[q];
        const double d = v.x - xr;
        const double w = ll_weight<KERN>(fabs(d), h);
        s0 += w;
        sd = fma(w, d, sd);
        sy = fma(w, v.y, sy);
    }
    const double dbar = sd / s0, ybar = sy / s0;
    double sdd = 0.0, sdy = 0.0;
    for (int q = A; q < R; q++) {
        if (q == r) continue;
        const double2 v = xy[q];
        const double d = v.x - xr;
        const double w = ll_weight<KERN>(fabs(d), h);
        const double dc = d - dbar;
        const double wdc = w * dc;
        sdd = fma(wdc, dc, sdd);
        sdy = fma(wdc, v.y - ybar, sdy);
    }
    return ybar - dbar * (sdy / sdd);
}

// Shifted power sums over [a, b) in dd: D[k] = sum (u - delta)^k
// (k = 1..DU) and Y[k] = sum y (u - delta)^k (k = 0..DY; Y[0] minus ysub),
// with absolute error bounds
// eD[k], eY[k] = kappa sum_i C(k,i) |delta|^(k-i) (|P_i[a]| + |P_i[b]|).
// Slots (kLLMoments): 0 y, 1 u, 2 u^2, 3 u^3, 4 u^4, 5 y u, 6 y u^2, 7 y u^3.
template <int DU, int DY>
__device__ __forceinline__ void ll_shift(const double *__restrict__ P, int ps, int a, int b, dd del, double ysub,
                                         double kappa, dd (&D)[5], dd (&Y)[4], double (&eD)[5], double (&eY)[4])
{
    const dd e = dd_neg(del);
    const double ad = fabs(del.hi);
    dd Mu[5], My[4];
    double au[5], ay[4];
    Mu[0] = dd_make((double)(b - a));
    au[0] = (double)(b - a);  // exact, but the Horner intermediates reach c' |delta|^k
#pragma unroll
    for (int k = 1; k <= DU; k++) {
        const dd pb = ld_pdd(P, ps, k, b), pa = ld_pdd(P, ps, k, a);
        Mu[k] = dd_sub(pb, pa);
        au[k] = fabs(pb.hi) + fabs(pa.hi);
    }
#pragma unroll
    for (int k = 0; k <= DY; k++) {
        const int slot = k == 0 ? 0 : 4 + k;
        const dd pb = ld_pdd(P, ps, slot, b), pa = ld_pdd(P, ps, slot, a);
        My[k] = dd_sub(pb, pa);
        ay[k] = fabs(pb.hi) + fabs(pa.hi);
    }
    // D_k = sum_i C(k,i) Mu_i e^(k-i): Horner in e (and in |delta| for the bound)
#pragma unroll
    for (int k = 1; k <= DU; k++) {
        dd acc = Mu[0];
        double mag = au[0];
        double cb = 1.0;
#pragma unroll
        for (int i = 1; i <= k; i++) {
            cb = cb * (double)(k - i + 1) / (double)i;
            acc = dd_add(dd_mul_d_raw(Mu[i], cb), dd_mul_raw(e, acc));
            mag = fma(cb, au[i], ad * mag);
        }
        D[k] = acc;
        eD[k] = kappa * mag;
    }
#pragma unroll
    for (int k = 0; k <= DY; k++) {
        dd acc = My[0];
        double mag = ay[0];
        double cb = 1.0;
#pragma unroll
        for (int i = 1; i <= k; i++) {
            cb = cb * (double)(k - i + 1) / (double)i;
            acc = dd_add(dd_mul_d_raw(My[i], cb), dd_mul_raw(e, acc));
            mag = fma(cb, ay[i], ad * mag);
        }
        if (k == 0) acc = dd_add_d(acc, -ysub);
        Y[k] = acc;
        eY[k] = kappa * mag;
    }
}

// H a - b in dd (H, a, b dd): the S_k / T_k of the weighted sums
__device__ __forceinline__ dd ll_comb(dd H, dd a, dd b) { return dd_sub(dd_mul(H, a), b); }

// Plain-double fast path (uniform / Epanechnikov): the hi words of P only,
// the binomial shift, S, T, det and num in double, with a bound of the same
// form as the dd path's -- every prefix value carries <= 2^-53 relative
// rounding (its dd lo part dropped), every Horner / fma step <= 2^-53 of the
// magnitude it combines (kf = 2^-49 covers them with slack), and delta's own
// rounding (only del.hi is used) shifts each d by |del.lo|, changing
// sum d^k by <= k |del.lo| c' h^(k-1).  Returns false when the bound is not
// below the dd path's tolerance (the caller then takes the dd path).
template <int KERN>
__device__ __forceinline__ bool ll_fast(const WinRow &w, int A, int R, int c, double h,
                                        const double *__restrict__ P, int ps, double ymax, double &g)
{
    constexpr int DU = KERN == KR_UNIFORM ? 2 : 4, DY = KERN == KR_UNIFORM ? 1 : 3;
    const double kf = 0x1p-49;
    const double e = -w.del.hi, ad = fabs(w.del.hi), dlo = fabs(w.del.lo);
    const double c1 = (double)(c + 1);  // points in [A, R), row r included
    double U[5], aU[5], Yr[4], aY[4];
    U[0] = c1;
    aU[0] = c1;  // exact, but the Horner intermediates reach c' |delta|^k
#pragma unroll
    for (int k = 1; k <= DU; k++) {
        const double pb = ld_hi(P, ps, k, R), pa = ld_hi(P, ps, k, A);
        U[k] = pb - pa;
        aU[k] = fabs(pb) + fabs(pa);
    }
#pragma unroll
    for (int k = 0; k <= DY; k++) {
        const int slot = k == 0 ? 0 : 4 + k;
        const double pb = ld_hi(P, ps, slot, R), pa = ld_hi(P, ps, slot, A);
        Yr[k] = pb - pa;
        aY[k] = fabs(pb) + fabs(pa);
    }
    double D[5], eD[5], Y[4], eY[4];
    double hp = 1.0;  // h^(k-1)
#pragma unroll
    for (int k = 1; k <= DU; k++) {
        double acc = U[0], mag = aU[0], cb = 1.0;
#pragma unroll
        for (int i = 1; i <= k; i++) {
            cb = cb * (double)(k - i + 1) / (double)i;
            acc = fma(acc, e, cb * U[i]);
            mag = fma(mag, ad, cb * aU[i]);
        }
        D[k] = acc;
        eD[k] = fma(kf, mag + fabs(acc), 2.0 * k * dlo * c1 * hp);
        hp *= h;
    }
    hp = 1.0;
    const double ay0 = c1 * ymax;
#pragma unroll
    for (int k = 0; k <= DY; k++) {
        double acc = Yr[0], mag = aY[0], cb = 1.0;
#pragma unroll
        for (int i = 1; i <= k; i++) {
            cb = cb * (double)(k - i + 1) / (double)i;
            acc = fma(acc, e, cb * Yr[i]);
            mag = fma(mag, ad, cb * aY[i]);
        }
        if (k == 0) {  // LOO: drop row r's own y
            acc -= w.yr;
            mag += fabs(w.yr);
        }
        Y[k] = acc;
        eY[k] = fma(kf, mag + fabs(acc), k > 0 ? 2.0 * k * dlo * ay0 * hp : 0.0);
        if (k > 0) hp *= h;
    }
    double S0, S1, S2, T0, T1, eS0, eS1, eS2, eT0, eT1;
    const double q = 0x1p-52;
    if (KERN == KR_UNIFORM) {
        S0 = (double)c; S1 = D[1]; S2 = D[2]; T0 = Y[0]; T1 = Y[1];
        eS0 = 0.0; eS1 = eD[1]; eS2 = eD[2]; eT0 = eY[0]; eT1 = eY[1];
    } else {
        const double hh = h * h;
        S0 = fma(hh, (double)c, -D[2]);
        S1 = fma(hh, D[1], -D[3]);
        S2 = fma(hh, D[2], -D[4]);
        T0 = fma(hh, Y[0], -Y[2]);
        T1 = fma(hh, Y[1], -Y[3]);
        // hh's rounding (q hh |.|), the fma's (q |result|), the inputs' bounds
        eS0 = eD[2] + q * (hh * (double)c + fabs(S0));
        eS1 = fma(hh, eD[1], eD[3]) + q * (hh * fabs(D[1]) + fabs(S1));
        eS2 = fma(hh, eD[2], eD[4]) + q * (hh * fabs(D[2]) + fabs(S2));
        eT0 = fma(hh, eY[0], eY[2]) + q * (hh * fabs(Y[0]) + fabs(T0));
        eT1 = fma(hh, eY[1], eY[3]) + q * (hh * fabs(Y[1]) + fabs(T1));
    }
    const double s11 = S1 * S1, s1t1 = S1 * T1;
    const double dt = fma(S0, S2, -s11), nm = fma(S2, T0, -s1t1);
    g = nm / dt;
    const double aS0 = fabs(S0), aS1 = fabs(S1), aS2 = fabs(S2), aT0 = fabs(T0), aT1 = fabs(T1);
    const double edet = aS2 * eS0 + aS0 * eS2 + 2.0 * aS1 * eS1 + eS0 * eS2 + eS1 * eS1 +
                        q * (aS0 * aS2 + s11 + fabs(dt));
    const double enum_ = aS2 * eT0 + aT0 * eS2 + aS1 * eT1 + aT1 * eS1 + eS2 * eT0 + eS1 * eT1 +
                         q * (aS2 * aT0 + fabs(s1t1) + fabs(nm));
    return dt > 0.0 && edet <= 0x1p-20 * dt && fma(fabs(g), edet, enum_) <= 0x1p-44 * dt * ymax;
}

// Local-linear g for row r, window [A, R) (c = R - A - 1 >= 2 points besides
// r, at least two distinct x).  S_k, T_k, det and num stay in dd; the error
// bounds eS, eT propagate the prefix errors, and dd rounding adds
// 2^-100 of the magnitudes combined.  Returns g.
template <int KERN>
__device__ __forceinline__ double ll_estimate(const WinRow &w, int A, int R, int c, double h,
                                              const double2 *__restrict__ xy, const double *__restrict__ P, int ps,
                                              double ymax, double kappa,
                                              unsigned long long *__restrict__ stats)
{
    const int r = w.r;
    if (c <= kLLDirect) {
        if (stats) atomicAdd(stats + 0, 1ull);
        return ll_direct<KERN>(xy, A, R, r, w.xr, h);
    }
    if (KERN != KR_TRIANGULAR) {
        double gf;
        if (ll_fast<KERN>(w, A, R, c, h, P, ps, ymax, gf)) {
            if (stats) atomicAdd(stats + 1, 1ull);
            return gf;
        }
    }
    dd S0, S1, S2, T0, T1;
    double eS0, eS1, eS2, eT0, eT1;
    const dd cc = dd_make((double)c);
    if (KERN != KR_TRIANGULAR) {
        dd D[5], Y[4];
        double eD[5], eY[4];
        // row r is inside [A, R): its d-terms vanish, its y leaves Y_0 (LOO)
        if (KERN == KR_UNIFORM) {
            ll_shift<2, 1>(P, ps, A, R, w.del, w.yr, kappa, D, Y, eD, eY);
            S0 = cc; S1 = D[1]; S2 = D[2]; T0 = Y[0]; T1 = Y[1];
            eS0 = 0.0; eS1 = eD[1]; eS2 = eD[2]; eT0 = eY[0]; eT1 = eY[1];
        } else {
            ll_shift<4, 3>(P, ps, A, R, w.del, w.yr, kappa, D, Y, eD, eY);
            const dd H = two_prod(h, h);  // h^2 exactly
            const double hh = H.hi;
            S0 = ll_comb(H, cc, D[2]);
            S1 = ll_comb(H, D[1], D[3]);
            S2 = ll_comb(H, D[2], D[4]);
            T0 = ll_comb(H, Y[0], Y[2]);
            T1 = ll_comb(H, Y[1], Y[3]);
            eS0 = eD[2];
            eS1 = fma(hh, eD[1], eD[3]);
            eS2 = fma(hh, eD[2], eD[4]);
            eT0 = fma(hh, eY[0], eY[2]);
            eT1 = fma(hh, eY[1], eY[3]);
        }
    } else {
        dd DR[5], YR[4], DL[5], YL[4];
        double eDR[5], eYR[4], eDL[5], eYL[4];
        ll_shift<3, 2>(P, ps, r + 1, R, w.del, 0.0, kappa, DR, YR, eDR, eYR);  // row r in neither part
        ll_shift<3, 2>(P, ps, A, r, w.del, 0.0, kappa, DL, YL, eDL, eYL);
        // right d = |d|, left d = -|d|: sum |d|^k = DR_k + (-1)^k DL_k
        const dd H = dd_make(h);
        S0 = ll_comb(H, cc, dd_sub(DR[1], DL[1]));
        S1 = ll_comb(H, dd_add(DR[1], DL[1]), dd_sub(DR[2], DL[2]));
        S2 = ll_comb(H, dd_add(DR[2], DL[2]), dd_sub(DR[3], DL[3]));
        T0 = ll_comb(H, dd_add(YR[0], YL[0]), dd_sub(YR[1], YL[1]));
        T1 = ll_comb(H, dd_add(YR[1], YL[1]), dd_sub(YR[2], YL[2]));
        eS0 = eDR[1] + eDL[1];
        eS1 = fma(h, eDR[1] + eDL[1], eDR[2] + eDL[2]);
        eS2 = fma(h, eDR[2] + eDL[2], eDR[3] + eDL[3]);
        eT0 = fma(h, eYR[0] + eYL[0], eYR[1] + eYL[1]);
        eT1 = fma(h, eYR[1] + eYL[1], eYR[2] + eYL[2]);
    }
    // det = S0 S2 - S1^2 and num = S2 T0 - S1 T1 in dd (they cancel when the
    // window sits far to one side of the row)
    const dd det = dd_sub(dd_mul(S0, S2), dd_mul(S1, S1));
    const dd num = dd_sub(dd_mul(S2, T0), dd_mul(S1, T1));
    const double dt = dd_to_d(det), nm = dd_to_d(num);
    const double g = nm / dt;
    // first-order propagation of eS, eT plus dd rounding (2^-100 relative to
    // the products, generously)
    const double aS0 = fabs(S0.hi), aS1 = fabs(S1.hi), aS2 = fabs(S2.hi);
    const double aT0 = fabs(T0.hi), aT1 = fabs(T1.hi);
    const double q = 0x1p-100;
    const double fS0 = fma(q, aS0, eS0), fS1 = fma(q, aS1, eS1), fS2 = fma(q, aS2, eS2);
    const double fT0 = fma(q, aT0, eT0), fT1 = fma(q, aT1, eT1);
    const double edet = aS2 * fS0 + aS0 * fS2 + 2.0 * aS1 * fS1 + fS0 * fS2 + fS1 * fS1 + q * (aS0 * aS2 + aS1 * aS1);
    const double enum_ =
        aS2 * fT0 + aT0 * fS2 + aS1 * fT1 + aT1 * fS1 + fS2 * fT0 + fS1 * fT1 + q * (aS2 * aT0 + aS1 * aT1);
    const bool ok = dt > 0.0 && edet <= 0x1p-20 * dt && fma(fabs(g), edet, enum_) <= 0x1p-44 * dt * ymax;
    if (stats) {
        atomicAdd(stats + (ok ? 1 : 2), 1ull);
        if (!ok) atomicAdd(stats + 3, (unsigned long long)c);
    }
    if (ok) return g;
    return ll_direct<KERN>(xy, A, R, r, w.xr, h);
}

// A warp owns 32 consecutive sorted rows (one per lane) and a chunk of the
// bandwidth loop, as window_kernel<KERN, 1>; output in the same tile-partial
// layout (reduce_kernel and the finalize are shared with Nadaraya-Watson).
// stats (debug, nullable): counts of direct / prefix-accepted (fast double
// or dd) / prefix-rejected (row, bandwidth) evaluations and the rejected
// windows' total size.
template <int KERN>
__global__ void __launch_bounds__(kWinThreads)
ll_window_kernel(const double *__restrict__ xs, const double2 *__restrict__ xy, const double *__restrict__ P,
                 int pstride, const double *__restrict__ hg, int m, int n, int row_lo, int row_hi, int ntiles,
                 int nbc, const unsigned long long *__restrict__ ymax_bits, double *__restrict__ tileS,
                 uint8_t *__restrict__ tileN, int *__restrict__ tile_counter,
                 unsigned long long *__restrict__ stats)
{
    const int lane = threadIdx.x & 31;
    const double o = pfx_origin(xy, n);
    const double ymax = __longlong_as_double((long long)*ymax_bits);
    const double kappa = ((double)n + 64.0) * 0x1p-104 + 0x1p-100;
    const int bper = (m + nbc - 1) / nbc;
    const int ps = pstride;
    for (;;) {
        int task = 0;
        if (lane == 0) task = atomicAdd(tile_counter, 1);
        task = __shfl_sync(0xffffffffu, task, 0);
        if (task >= ntiles * nbc) return;  // warp-uniform
        const int chunk = task / ntiles;   // chunk-major (see window_kernel)
        const int tile = task - chunk * ntiles;
        const int b0 = chunk * bper, b1 = min(m, b0 + bper);
        const int i = row_lo + tile * 32 + lane;
        const bool valid = i < row_hi;
        WinRow row;
        row.r = valid ? i : row_hi - 1;
        {
            const double2 v = xy[row.r];
            row.xr = v.x;
            row.yr = v.y;
            row.del = two_sum(v.x, -o);
        }
        int kR = 1, kL = 1, gR = cold_step(xs, n, __ldg(hg + b0)), gL = gR;
        for (int b = b0; b < b1; b++) {
            const double h = __ldg(hg + b);
            const int kR0 = kR, kL0 = kL;
            window_bounds<KERN>(xs, n, row.r, row.xr, h, kR, kL, gR, gL);
            gR = max(1, kR - kR0);
            gL = max(1, kL - kL0);
            const int R = row.r + kR, A = row.r - kL + 1;
            const int c = R - A - 1;
            double e2 = 0.0;
            int cntM = 0;
            if (valid && c >= 2) {
                // reading Q25: >= 2 distinct x among the window's points (sorted:
                // compare the first and the last, skipping the row itself)
                const int first = A == row.r ? A + 1 : A;
                const int last = R - 1 == row.r ? R - 2 : R - 1;
                if (xs[first] != xs[last]) {
                    const double g = ll_estimate<KERN>(row, A, R, c, h, xy, P, ps, ymax, kappa, stats);
                    const double e = row.yr - g;
                    e2 = e * e;
                    cntM = 1;
                }
            }
            e2 = warp_sum(e2);
            const int cnt = __reduce_add_sync(0xffffffffu, cntM);
            if (lane == 0) {
                tileS[(size_t)b * ntiles + tile] = e2;
                tileN[(size_t)b * ntiles + tile] = (uint8_t)cnt;
            }
        }
    }
}

}  // namespace krcv
