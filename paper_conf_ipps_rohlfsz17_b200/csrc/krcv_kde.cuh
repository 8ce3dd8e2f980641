// krcv_kde.cuh -- KDE least-squares cross-validation (
// PAPER.md P@10382-10640 "the methods developed here for least-squares
// cross-validation can be applied to ... optimal bandwidth selection for
// kernel density estimation"; reading Q24).
//
//   LSCV(h) = (n Kbar(0) + sum_i A_i) / (n^2 h) - 2 sum_i B_i / (n (n-1) h)
//   A_i = sum_{j!=i, |d|<2h} Kbar(d/h),  B_i = sum_{j!=i, d in K's window} K(d/h)
//
// Kbar = K * K and K are polynomials in v = |d|/h on their windows, so the
// same machinery as the regression's window-prefix path applies: the sorted
// x, galloping boundary searches with the exact binary64 predicates (K's
// window, reading Q1, and |d| < 2h for Kbar), and double-double prefix sums
// of u^k (u = x - o, k = 1..5).  Odd powers of |d| split the window at the
// row (right: d = u - delta, left: |d| = delta - u); the power sums about the
// row follow from the raw ones by the binomial shift
//   T_k = sum_{(r,R)} (u - delta)^k = sum_i C(k,i) M_i (-delta)^(k-i)
// evaluated in dd.  Per (row, bandwidth) the Epanechnikov kernel needs
// c, S2 on K's window and c, S2, S3, S5 on Kbar's (S_k = sum |d|^k):
//   B = 3/4 (c1 - S2_1/h^2)
//   A = 3/160 (32 c2 - 40 S2_2/h^2 + 20 S3_2/h^3 - S5_2/h^5)
// uniform: B = c1/2, A = (2 c2 - S1_2/h)/4; triangular: B = c1 - S1_1/h,
// A = [2/3 c1 - S2_1/h^2 + S3_1/(2h^3)]                          (|v| < 1)
//   + [8 dc - 12 dS1/h + 6 dS2/h^2 - dS3/h^3] / 6   (1 <= |v| < 2, d* = W2 - W1).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "krcv.h"
#include "krcv_dd.cuh"
#include "krcv_prefix.cuh"

namespace krcv {

// Power sums of |d| over the right part (r, R) and the left part [A, r) of a
// window, k = 1..DEG, from the KDE prefix planes (moment k-1 holds u^k).
// S[k] = sum_right (u - delta)^k + (-1)^k sum_left (u - delta)^k = sum |d|^k.
template <int DEG>
__device__ __forceinline__ void kde_power_sums(const double *__restrict__ P, int ps, int r, int A, int R, dd del,
                                               double (&S)[6])
{
    const dd e = dd_neg(del);
    dd TR[6], TL[6];
#pragma unroll
    for (int side = 0; side < 2; side++) {
        const int a = side == 0 ? r + 1 : A, b = side == 0 ? R : r;
        dd M[6];
        M[0] = dd_make((double)(b - a));
#pragma unroll
        for (int k = 1; k <= DEG; k++) M[k] = wsum(P, ps, k - 1, a, b);
        dd *T = side == 0 ? TR : TL;
        // T_k = sum_i C(k,i) M_i e^(k-i), Horner in e
#pragma unroll
        for (int k = 1; k <= DEG; k++) {
            if (DEG == 5 && k == 4) continue;  // S4 is never needed
            dd acc = M[0];
            double cbin = 1.0;  // C(k, i) for i = 0 .. k, built incrementally
#pragma unroll
            for (int i = 1; i <= k; i++) {
                cbin = cbin * (double)(k - i + 1) / (double)i;
                acc = dd_add(dd_mul_d_raw(M[i], cbin), dd_mul_raw(e, acc));
            }
            T[k] = acc;
        }
    }
#pragma unroll
    for (int k = 1; k <= DEG; k++) {
        if (DEG == 5 && k == 4) continue;
        S[k] = dd_to_d((k & 1) ? dd_sub(TR[k], TL[k]) : dd_add(TR[k], TL[k]));
    }
}

// Plain-double fast path of kde_power_sums (hi words of P only, Horner in
// double) with a rigorous bound of its error.  Each raw moment difference
// M_i = P_hi[b] - P_hi[a] is off by at most 2^-52 (|P_hi[b]| + |P_hi[a]|)
// (hi word rounding of the dd prefix + the subtraction); Horner's 2k roundings
// and the rounding of delta (k 2^-53 relative, first order) are bounded by
// the same binomial sum of magnitudes E_k = sum_i C(k,i) Mb_i |delta|^(k-i),
// so |S_k - S_k(fast)| <= (3k + 4) 2^-52 (E_k right + E_k left) (twice the
// first-order estimate: the magnitudes are themselves rounded).  Empty sides
// contribute exactly 0 (P_hi[b] == P_hi[a]) and no error.
template <int DEG>
__device__ __forceinline__ void kde_power_sums_fast(const double *__restrict__ P, int ps, int r, int A, int R,
                                                    double dl, double (&S)[6], double (&err)[6])
{
    const double e = -dl, ae = fabs(dl);
    double TR[6], TL[6], ER[6], EL[6];
#pragma unroll
    for (int side = 0; side < 2; side++) {
        const int a = side == 0 ? r + 1 : A, b = side == 0 ? R : r;
        const bool empty = b <= a;
        double M[6], Mb[6];
        M[0] = empty ? 0.0 : (double)(b - a);
        Mb[0] = M[0];
#pragma unroll
        for (int k = 1; k <= DEG; k++) {
            const double pb = ld_hi(P, ps, k - 1, b), pa = ld_hi(P, ps, k - 1, a);
            M[k] = empty ? 0.0 : pb - pa;
            Mb[k] = empty ? 0.0 : fabs(pb) + fabs(pa);
        }
        double *T = side == 0 ? TR : TL;
        double *E = side == 0 ? ER : EL;
#pragma unroll
        for (int k = 1; k <= DEG; k++) {
            if (DEG == 5 && k == 4) continue;  // S4 is never needed
            double acc = M[0], mag = Mb[0], cbin = 1.0;
#pragma unroll
            for (int i = 1; i <= k; i++) {
                cbin = cbin * (double)(k - i + 1) / (double)i;  // exact small integers
                acc = fma(e, acc, cbin * M[i]);
                mag = fma(ae, mag, cbin * Mb[i]);
            }
            T[k] = acc;
            E[k] = mag;
        }
    }
#pragma unroll
    for (int k = 1; k <= DEG; k++) {
        if (DEG == 5 && k == 4) continue;
        S[k] = (k & 1) ? TR[k] - TL[k] : TR[k] + TL[k];
        err[k] = (3.0 * k + 4.0) * 0x1p-52 * (ER[k] + EL[k]);
    }
}

// Fast results are kept when the bound on the error of A_i (B_i) is below
// kKdeFastTol times the largest value A_i (B_i) can take, c Kbar(0) (c K(0)):
// per row an absolute error <= 2^-44 of its possible contribution.
constexpr double kKdeFastTol = 0x1p-44;

template <int KERN>
__global__ void __launch_bounds__(kWinThreads)
kde_window_kernel(const double *__restrict__ xs, const double2 *__restrict__ xy, const double *__restrict__ P,
                  int pstride, const double *__restrict__ hg, int m, int n, int row_lo, int row_hi, int ntiles,
                  int nbc, double *__restrict__ tileA, double *__restrict__ tileB, int *__restrict__ tile_counter)
{
    const int lane = threadIdx.x & 31;
    const double o = pfx_origin(xy, n);
    const int bper = (m + nbc - 1) / nbc;
    const int ps = pstride;
    for (;;) {
        int task = 0;
        if (lane == 0) task = atomicAdd(tile_counter, 1);
        task = __shfl_sync(0xffffffffu, task, 0);
        if (task >= ntiles * nbc) return;  // warp-uniform
        const int chunk = task / ntiles;  // chunk-major (see window_kernel)
        const int tile = task - chunk * ntiles;
        const int b0 = chunk * bper, b1 = min(m, b0 + bper);
        const int i = row_lo + tile * 32 + lane;
        const bool valid = i < row_hi;
        const int r = valid ? i : row_hi - 1;
        const double xr = xy[r].x;
        const dd del = two_sum(xr, -o);  // exact x_r - o
        int kR1 = 1, kL1 = 1, gR1 = cold_step(xs, n, __ldg(hg + b0)), gL1 = gR1;  // K's window (radius h)
        int kR2 = 1, kL2 = 1, gR2 = 2 * gR1, gL2 = gR2;  // Kbar's window (radius 2h, open)
        for (int b = b0; b < b1; b++) {
            const double h = __ldg(hg + b), h2 = 2.0 * h;  // 2h exact
            {
                const int a0 = kR1, c0 = kL1;
                window_bounds<KERN>(xs, n, r, xr, h, kR1, kL1, gR1, gL1);
                gR1 = max(1, kR1 - a0);
                gL1 = max(1, kL1 - c0);
            }
            {
                const int a0 = kR2, c0 = kL2;
                window_bounds<KR_EPANECHNIKOV>(xs, n, r, xr, h2, kR2, kL2, gR2, gL2);  // open: |d| < 2h
                gR2 = max(1, kR2 - a0);
                gL2 = max(1, kL2 - c0);
            }
            const int R1 = r + kR1, A1 = r - kL1 + 1, R2 = r + kR2, A2 = r - kL2 + 1;
            const double c1 = (double)(R1 - A1 - 1), c2 = (double)(R2 - A2 - 1);
            const double ih = 1.0 / h, ih2 = ih * ih, ih3 = ih2 * ih;
            double Ai, Bi;
            if (KERN == KR_UNIFORM) {  // one power sum: dd directly (the fast path measured slower here)
                double S[6];
                kde_power_sums<1>(P, ps, r, A2, R2, del, S);
                Bi = 0.5 * c1;
                Ai = 0.25 * fma(-S[1], ih, 2.0 * c2);
            } else if (KERN == KR_EPANECHNIKOV) {
                double S1[6], S2[6], e1[6], e2[6];
                const double ih5 = ih3 * ih2;
                kde_power_sums_fast<2>(P, ps, r, A1, R1, del.hi, S1, e1);
                kde_power_sums_fast<5>(P, ps, r, A2, R2, del.hi, S2, e2);
                const double errB = 0.75 * e1[2] * ih2;
                const double errA = (3.0 / 160.0) * (40.0 * e2[2] * ih2 + 20.0 * e2[3] * ih3 + e2[5] * ih5 +
                                                     8.0 * 0x1p-53 * (32.0 * c2 + 40.0 * fabs(S2[2]) * ih2 +
                                                                      20.0 * fabs(S2[3]) * ih3 + fabs(S2[5]) * ih5));
                if (!(errB <= kKdeFastTol * 0.75 * c1)) kde_power_sums<2>(P, ps, r, A1, R1, del, S1);
                if (!(errA <= kKdeFastTol * 0.6 * c2)) kde_power_sums<5>(P, ps, r, A2, R2, del, S2);
                Bi = 0.75 * fma(-S1[2], ih2, c1);
                Ai = (3.0 / 160.0) * (32.0 * c2 - 40.0 * S2[2] * ih2 + 20.0 * S2[3] * ih3 - S2[5] * ih5);
            } else {
                double S1[6], S2[6], e1[6], e2[6];
                kde_power_sums_fast<3>(P, ps, r, A1, R1, del.hi, S1, e1);
                kde_power_sums_fast<3>(P, ps, r, A2, R2, del.hi, S2, e2);
                const double errB = e1[1] * ih;
                const double errA = e1[2] * ih2 + 0.5 * e1[3] * ih3 +
                                    (12.0 * (e2[1] + e1[1]) * ih + 6.0 * (e2[2] + e1[2]) * ih2 +
                                     (e2[3] + e1[3]) * ih3) / 6.0 +
                                    8.0 * 0x1p-53 * (c1 + c2 + (fabs(S2[1]) + fabs(S1[1])) * 2.0 * ih +
                                                     (fabs(S2[2]) + fabs(S1[2])) * ih2 +
                                                     (fabs(S2[3]) + fabs(S1[3])) * ih3);
                if (!(errB <= kKdeFastTol * c1 && errA <= kKdeFastTol * (2.0 / 3.0) * c2)) {
                    kde_power_sums<3>(P, ps, r, A1, R1, del, S1);
                    kde_power_sums<3>(P, ps, r, A2, R2, del, S2);
                }
                Bi = fma(-S1[1], ih, c1);
                const double inner = (2.0 / 3.0) * c1 - S1[2] * ih2 + 0.5 * S1[3] * ih3;
                const double outer = (8.0 * (c2 - c1) - 12.0 * (S2[1] - S1[1]) * ih + 6.0 * (S2[2] - S1[2]) * ih2 -
                                      (S2[3] - S1[3]) * ih3) / 6.0;
                Ai = inner + outer;
            }
            if (!valid) {
                Ai = 0.0;
                Bi = 0.0;
            }
            Ai = warp_sum(Ai);
            Bi = warp_sum(Bi);
            if (lane == 0) {
                tileA[(size_t)b * ntiles + tile] = Ai;
                tileB[(size_t)b * ntiles + tile] = Bi;
            }
        }
    }
}

// Fixed-order column sums -> partial [sum A | sum B | status]; with lscv set
// the last CTA also finalizes (as reduce_kernel).
struct KdeFin {
    long long n;
    int kernel;
    const double *h;
    double *lscv;
    int *best, *status;
    unsigned *done;
};

constexpr int kKdeRedThreads = 256;

__global__ void __launch_bounds__(kKdeRedThreads)
kde_reduce_kernel(const double *__restrict__ tileA, const double *__restrict__ tileB, int ntiles, int m,
                  const unsigned *__restrict__ status, double *__restrict__ partial, KdeFin fin)
{
    __shared__ double sA[kKdeRedThreads], sB[kKdeRedThreads];
    __shared__ int sI[kKdeRedThreads];
    __shared__ bool last;
    for (int b = blockIdx.x; b < m; b += gridDim.x) {
        double a = 0.0, c = 0.0;
        for (int t = threadIdx.x; t < ntiles; t += kKdeRedThreads) {
            a += tileA[(size_t)b * ntiles + t];
            c += tileB[(size_t)b * ntiles + t];
        }
        sA[threadIdx.x] = a;
        sB[threadIdx.x] = c;
        __syncthreads();
        for (int s = kKdeRedThreads / 2; s > 0; s >>= 1) {
            if (threadIdx.x < s) {
                sA[threadIdx.x] += sA[threadIdx.x + s];
                sB[threadIdx.x] += sB[threadIdx.x + s];
            }
            __syncthreads();
        }
        if (threadIdx.x == 0) {
            partial[b] = sA[0];
            partial[m + b] = sB[0];
        }
        __syncthreads();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        partial[2 * m] = (double)status[0];
        partial[2 * m + 1] = (double)status[1];
    }
    if (fin.lscv == nullptr) return;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last = atomicAdd(fin.done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!last) return;
    __threadfence();
    // LSCV(h_b) = (n Kbar(0) + A) / (n^2 h) - 2 B / (n (n-1) h); arg-min per Q11
    const double nn = (double)fin.n;
    const double kb0 = fin.kernel == KR_UNIFORM ? 0.5 : (fin.kernel == KR_EPANECHNIKOV ? 0.6 : 2.0 / 3.0);
    double bv = 0.0;
    int bi = -1;
    for (int b = threadIdx.x; b < m; b += kKdeRedThreads) {
        const double hb = __ldg(fin.h + b);
        const double v = (nn * kb0 + __ldcg(partial + b)) / (nn * nn * hb) -
                         2.0 * __ldcg(partial + m + b) / (nn * (nn - 1.0) * hb);
        fin.lscv[b] = v;
        if (!isnan(v) && (bi < 0 || v < bv)) {
            bv = v;
            bi = b;
        }
    }
    sA[threadIdx.x] = bv;
    sI[threadIdx.x] = bi;
    __syncthreads();
    for (int s = kKdeRedThreads / 2; s > 0; s >>= 1) {
        if (threadIdx.x < s) {
            const double ov = sA[threadIdx.x + s], mv = sA[threadIdx.x];
            const int oi = sI[threadIdx.x + s], mi = sI[threadIdx.x];
            if (oi >= 0 && (mi < 0 || ov < mv || (ov == mv && oi < mi))) {
                sA[threadIdx.x] = ov;
                sI[threadIdx.x] = oi;
            }
        }
        __syncthreads();
    }
    if (threadIdx.x == 0) {
        *fin.best = sI[0] < 0 ? 0 : sI[0];
        int st = KR_OK;
        if (__ldcg(partial + 2 * m) != 0.0) st = KR_EGRID;
        else if (__ldcg(partial + 2 * m + 1) != 0.0) st = KR_ENONFINITE;
        *fin.status = st;
        *fin.done = 0u;
    }
}

}  // namespace krcv
