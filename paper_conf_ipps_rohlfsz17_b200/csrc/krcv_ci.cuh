// krcv_ci.cuh -- leave-one-out (delete-one jackknife) confidence intervals at
// the cross-validated bandwidth (§II P@10560-10640: "the estimation
// of leave-one-out cross-validated confidence intervals for kernel density
// estimates and kernel regressions"; reading Q26,
// DESIGN.md §2 and §6.9).
//
// Runs after a grid search on the same workspace: the sorted (x, y) records,
// the permutation back to the caller's order and the optimal index best (on
// the device, written by the fused finalize) are already there, so h* =
// h[best] is read on the device -- no host round trip between the search and
// the intervals.  Per sorted point r (one lane each, 32 consecutive points per
// warp, so the lanes' windows overlap and their loads coalesce):
//
//   window W+_r = [A, R) at h* INCLUDING r (reading Q1's predicate), found by
//   a gallop from r and a bisection (exact; O(log |W+|) probes);
//
//   regression (Nadaraya-Watson, Eq.(2) with the point itself):
//     pass 1  D = sum w_j, N = sum w_j y_j over W+ (w = (h-d)(h+d)
//             Epanechnikov, h - d triangular, 1 uniform: Eq.(3) / Q13 up to
//             a constant factor, which cancels below), g = N / D;
//     pass 2  Delta_j = -w_j (y_j - g) / (D - w_j)  (= g^(-j) - g, the
//             delete-one change), s1 = sum Delta_j, s2 = sum Delta_j^2;
//             V = (n-1)/n (s2 - s1^2 / n), se = sqrt(V); NaN when W+ = {r}
//             (no estimate without r);
//   density (Q24's normalised kernels, k_j = K(d_j / h) / h):
//     pass 1  S = sum k_j over W+, f = S / n;
//     pass 2  q = sum (k_j - f)^2 over W+ + (n - |W+|) f^2 (the points outside
//             the window contribute k_j = 0), V = q / (n (n-1)).
//
// Both passes are direct sums over the contiguous window in fixed order
// (bit-reproducible), fp64.  Output est / se in the caller's original order.
#pragma once

#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>

#include "krcv.h"
#include "krcv_pdl.cuh"
#include "krcv_sweep.cuh"

namespace krcv {

constexpr int kCiThreads = 128;

// first k in (r, n] outside the window of x_r at h (right), first k in [0, r]
// inside (left): gallop from r, then bisect.  Reads the sorted records xy
// (+-inf sentinels; present after either sort path, whichever algorithm
// searched the grid).
template <int KERN>
__device__ __forceinline__ void ci_window(const double2 *__restrict__ xy, int n, int r, double xr, double h, int &A,
                                          int &R)
{
    auto X = [&](int k) { return __ldg(&xy[k].x); };
    int lo = r, hi, step = 1;  // right: xs[lo] inside (lo = r: d = 0), find first outside
    for (;;) {
        hi = min(r + step, n);
        if (!inside<KERN>(X(hi) - xr, h)) break;
        lo = hi;
        if (hi == n) break;  // unreachable: xs[n] = +inf is outside
        step <<= 1;
    }
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (inside<KERN>(X(mid) - xr, h)) lo = mid; else hi = mid;
    }
    R = hi;
    int in = r, out, st = 1;  // left: xs[in] inside, find last outside (xs[-1] = -inf)
    for (;;) {
        out = max(r - st, -1);
        if (!inside<KERN>(xr - X(out), h)) break;
        in = out;
        st <<= 1;
    }
    while (in - out > 1) {
        const int mid = (in + out) >> 1;
        if (inside<KERN>(xr - X(mid), h)) in = mid; else out = mid;
    }
    A = in;
}

// weight of a point at distance d (d in the window): the regression's
// unnormalised K (constants cancel) or the density's normalised K(d/h)/h
template <int KERN, bool KDE>
__device__ __forceinline__ double ci_weight(double d, double h, double inv_h)
{
    if (KDE) {
        const double u = d * inv_h;
        return (KERN == KR_EPANECHNIKOV ? 0.75 * (1.0 - u) * (1.0 + u) : (KERN == KR_TRIANGULAR ? 1.0 - u : 0.5)) *
               inv_h;
    }
    return KERN == KR_EPANECHNIKOV ? (h - d) * (h + d) : (KERN == KR_TRIANGULAR ? h - d : 1.0);
}

template <int KERN, bool KDE>
__global__ void __launch_bounds__(kCiThreads)
ci_kernel(const double2 *__restrict__ xy, const uint32_t *__restrict__ perm, int n,
          const double *__restrict__ hg, const int *__restrict__ best, double *__restrict__ est,
          double *__restrict__ se)
{
    pdl_wait();  // krcv_pdl.cuh
    const int r = blockIdx.x * kCiThreads + threadIdx.x;
    if (r >= n) return;
    const double h = hg[*best];
    const double inv_h = 1.0 / h;
    const double xr = xy[r].x;
    int A, R;
    ci_window<KERN>(xy, n, r, xr, h, A, R);
    const double nn = (double)n;
    double e, s;
    if (KDE) {
        double S = 0.0;
        for (int j = A; j < R; j++) S += ci_weight<KERN, true>(fabs(__ldg(&xy[j].x) - xr), h, inv_h);
        const double f = S / nn;
        double q = 0.0;
        for (int j = A; j < R; j++) {
            const double t = ci_weight<KERN, true>(fabs(__ldg(&xy[j].x) - xr), h, inv_h) - f;
            q = fma(t, t, q);
        }
        q = fma((nn - (double)(R - A)) * f, f, q);
        e = f;
        s = sqrt(q / (nn * (nn - 1.0)));
    } else {
        double D = 0.0, N = 0.0;
        for (int j = A; j < R; j++) {
            const double2 v = xy[j];
            const double w = ci_weight<KERN, false>(fabs(v.x - xr), h, inv_h);
            D += w;
            N = fma(w, v.y, N);
        }
        const double g = N / D;
        double s1 = 0.0, s2 = 0.0;
        bool ok = true;
        for (int j = A; j < R; j++) {
            const double2 v = xy[j];
            const double w = ci_weight<KERN, false>(fabs(v.x - xr), h, inv_h);
            const double rest = D - w;
            ok = ok && rest > 0.0;
            const double delta = -w * (v.y - g) / rest;
            s1 += delta;
            s2 = fma(delta, delta, s2);
        }
        e = g;
        s = ok ? sqrt((nn - 1.0) / nn * (s2 - s1 * s1 / nn)) : NAN;
    }
    const uint32_t i = perm[r];
    est[i] = e;
    se[i] = s;
}

}  // namespace krcv
