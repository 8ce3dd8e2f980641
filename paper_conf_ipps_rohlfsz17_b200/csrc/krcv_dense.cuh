// krcv_dense.cuh -- Gaussian-kernel grid search (SURVEY.md §8(f) rank 1,
// PAPER.md P@10203 "it is straightforward to add additional [kernel
// weighting functions]"; reading Q23).
//
// The Gaussian K(u) = exp(-u^2/2) has no compact support, so neither the
// sorted sweep nor the window prefix applies: every (row, neighbour,
// bandwidth) triple carries a weight.  This is the tiled all-pairs kernel:
//   * a CTA owns 128 consecutive sorted rows (one per thread) and a chunk of
//     kGB bandwidths, whose numerator / denominator accumulators live in
//     registers;
//   * it streams the sorted (x, y) records through shared memory in tiles of
//     kGTile (16 KB), all threads reading the same record per step
//     (broadcast LDS, no bank conflicts);
//   * weights are rescaled by the row's nearest-neighbour weight (Q23:
//     w = exp(-(d^2 - dmin^2) / (2 h^2)), an exact identity for Eq.(2)), so
//     the nearest neighbour has weight 1, the denominator is >= 1 and
//     M_i = 1 -- no underflow can produce 0/0;
//   * columns whose rescaled weight is below e^-64 for every row of the tile
//     and every bandwidth of the chunk (|x_j - x_r| >= sqrt(dmin_max^2 +
//     128 h_max^2)) are skipped: their total is < n e^-64 relative to the
//     denominator, far below fp64 rounding;
//   * exp is evaluated in fp64 on the FP64 pipe (2^k scaling + degree-12
//     Taylor on |r| <= ln2/2, truncation error < 2e-16).
// The LOO term j == r gets weight 0.  Per (row, column, bandwidth): 1 DMUL,
// the exp (17 FP64 ops), 1 DFMA, 1 DADD.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "krcv.h"
#include "krcv_sweep.cuh"

namespace krcv {

constexpr int kGThreads = 128;  // rows per CTA, one per thread
constexpr int kGB = 8;          // bandwidths per CTA (register accumulators)
constexpr int kGTile = 1024;    // (x, y) records staged per round: 16 KB
constexpr double kGTrunc = 64.0;

// e^{-x}, x >= 0 (clamped at 708: the result stays normal).  x log2(e) is
// rounded to k with the 1.5 * 2^52 trick (k in the low word), r = -x - k ln2
// in two FMA steps (Cody-Waite), e^r by Horner on the Taylor series to
// degree 12, times 2^k built in the exponent field.
__device__ __forceinline__ double exp_neg(double x)
{
    x = fmin(x, 708.0);
    const double kMagic = 6755399441055744.0;  // 1.5 * 2^52
    const double t = __fma_rn(-x, 1.4426950408889634, kMagic);
    const double kd = __dsub_rn(t, kMagic);
    const int k = __double2loint(t);
    double r = __fma_rn(kd, -6.93147180369123816490e-01, -x);
    r = __fma_rn(kd, -1.90821492927058770002e-10, r);
    double p = 2.08767569878680989792e-09;  // 1/12!
    p = __fma_rn(p, r, 2.50521083854417187751e-08);
    p = __fma_rn(p, r, 2.75573192239858906526e-07);
    p = __fma_rn(p, r, 2.75573192239858906526e-06);
    p = __fma_rn(p, r, 2.48015873015873015873e-05);
    p = __fma_rn(p, r, 1.98412698412698412698e-04);
    p = __fma_rn(p, r, 1.38888888888888888889e-03);
    p = __fma_rn(p, r, 8.33333333333333333333e-03);
    p = __fma_rn(p, r, 4.16666666666666666667e-02);
    p = __fma_rn(p, r, 1.66666666666666666667e-01);
    p = __fma_rn(p, r, 0.5);
    p = __fma_rn(p, r, 1.0);
    p = __fma_rn(p, r, 1.0);
    return __dmul_rn(p, __hiloint2double((k + 1023) << 20, 0));
}

// First index j in [0, n) with x_j >= v (UPPER: x_j > v) on the sorted x
// (the sentinels are outside [0, n)).
template <bool UPPER>
__device__ __forceinline__ int bound_x(const double2 *__restrict__ xy, int n, double v)
{
    int lo = 0, len = n;
    while (len > 0) {
        const int half = len >> 1;
        const double xv = xy[lo + half].x;
        if (UPPER ? xv <= v : xv < v) {
            lo += half + 1;
            len -= half + 1;
        } else {
            len = half;
        }
    }
    return lo;
}

__global__ void __launch_bounds__(kGThreads)
gauss_kernel(const double2 *__restrict__ xy, int n, const double *__restrict__ hg, int m, int row_lo, int row_hi,
             int nbc, int ntiles, double *__restrict__ tileS, uint8_t *__restrict__ tileN)
{
    __shared__ double2 col[kGTile];
    __shared__ double s_max[kGThreads / 32];
    __shared__ int s_range[2];
    const int rt = blockIdx.x / nbc, bc = blockIdx.x - rt * nbc;
    const int b0 = bc * kGB;
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int i = row_lo + rt * kGThreads + t;
    const bool valid = i < row_hi;
    const int r = valid ? i : row_hi - 1;  // clamped rows do identical work, discarded
    const double2 vr = xy[r];
    const double xr = vr.x, yr = vr.y;
    // nearest neighbour in the sorted order (xy[-1] = -inf, xy[n] = +inf)
    const double dmin = fmin(xr - xy[r - 1].x, xy[r + 1].x - xr);
    const double dmin2 = dmin * dmin;
    double c[kGB], num[kGB], den[kGB];
    double hmax = 0.0;
#pragma unroll
    for (int q = 0; q < kGB; q++) {
        const double h = __ldg(hg + min(b0 + q, m - 1));
        hmax = fmax(hmax, h);
        c[q] = 0.5 / (h * h);
        num[q] = 0.0;
        den[q] = 0.0;
    }
    // column range that can matter for any row of the tile and bandwidth of
    // the chunk
    double dm = valid ? dmin2 : 0.0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dm = fmax(dm, __shfl_xor_sync(0xffffffffu, dm, o));
    if (lane == 0) s_max[w] = dm;
    __syncthreads();
    if (t == 0) {
        double dmax2 = s_max[0];
        for (int q = 1; q < kGThreads / 32; q++) dmax2 = fmax(dmax2, s_max[q]);
        const int first = row_lo + rt * kGThreads;
        const int last = min(row_hi, first + kGThreads) - 1;
        const double D = sqrt(dmax2 + 2.0 * kGTrunc * hmax * hmax);
        s_range[0] = bound_x<false>(xy, n, xy[first].x - D);
        s_range[1] = bound_x<true>(xy, n, xy[last].x + D);
    }
    __syncthreads();
    const int jlo = s_range[0], jhi = s_range[1];

    for (int j0 = jlo; j0 < jhi; j0 += kGTile) {
        const int cnt = min(kGTile, jhi - j0);
        __syncthreads();  // previous tile consumed
        for (int q = t; q < cnt; q += kGThreads) col[q] = xy[j0 + q];
        __syncthreads();
        const int self = r - j0;
        for (int q = 0; q < cnt; q++) {
            const double2 v = col[q];
            const double d = v.x - xr;
            const double tt = __fma_rn(d, d, -dmin2);
            const bool is_self = q == self;  // leave-one-out (Eq.(2) l != i)
#pragma unroll
            for (int k = 0; k < kGB; k++) {
                double wgt = exp_neg(tt * c[k]);
                wgt = is_self ? 0.0 : wgt;
                num[k] = __fma_rn(wgt, v.y, num[k]);
                den[k] += wgt;
            }
        }
    }

    const int tile = (rt * kGThreads + t) >> 5;  // 32-row tile of the partial layout
#pragma unroll
    for (int k = 0; k < kGB; k++) {
        const int b = b0 + k;
        if (b >= m) break;  // block-uniform
        const double e = yr - num[k] / den[k];
        double e2 = valid ? e * e : 0.0;
        e2 = warp_sum(e2);
        const unsigned ball = __ballot_sync(0xffffffffu, valid);
        if (lane == 0 && tile < ntiles) {
            tileS[(size_t)b * ntiles + tile] = e2;
            tileN[(size_t)b * ntiles + tile] = (uint8_t)__popc(ball);
        }
    }
}

}  // namespace krcv
