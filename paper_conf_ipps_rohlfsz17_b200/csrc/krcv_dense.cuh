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
//   * exp is evaluated in fp64 on the FP64 pipe: a 16-entry 2^(-j/16) table
//     in shared memory (conflict-free), Cody-Waite reduction, degree-7
//     Taylor (exp_neg_tab; the table-free exp_neg is kept as its reference).
// The LOO term j == r gets weight ~1e-304 (see the loop).  Per (row, column, bandwidth): 1 DMUL,
// the exp (13 FP64 ops + 1 LDS), 1 DFMA, 1 DADD.
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

// 2^(-j/16), j = 0..15, correctly rounded.  16 doubles = 128 B: staged in
// shared memory they occupy each of the 32 banks exactly once, so any
// per-lane index pattern is conflict-free (equal indices broadcast).
__device__ __constant__ double kExp2Tab[16] = {
    1.0, 0.9576032806985737, 0.9170040432046712, 0.8781260801866497,
    0.8408964152537145, 0.8052451659746271, 0.7711054127039704, 0.7384130729697497,
    0.7071067811865476, 0.6771277734684463, 0.6484197773255048, 0.620928906036742,
    0.5946035575013605, 0.5693943173783458, 0.5452538663326288, 0.5221368912137069};

// e^{-x} for 0 <= x <= 9e7, table-driven: N = round(16 x / ln2) (1.5 * 2^52
// trick, N in the low word: an int up to 2^31), r = x - N ln2/16
// (Cody-Waite, ln2/16 split so N * hi is exact), |r| <= ln2/32;
// e^{-x} = 2^{-(N>>4)} * 2^{-(N&15)/16} * e^{-r} with e^{-r} by the degree-7
// Taylor series (truncation < 1.3e-18).  The 2^{-(N>>4)} scaling subtracts
// from the table value's exponent field, N>>4 clamped at 1010 in the integer
// domain: for x > 700 the result is ~1e-304 instead of e^{-x}, i.e. zero next
// to the nearest-neighbour weight 1.  13 FP64-pipe ops + 1 conflict-free LDS
// (vs 18 FP64 for exp_neg).
__device__ __forceinline__ double exp_neg_tab(double x, const double *__restrict__ tab)
{
    const double kMagic = 6755399441055744.0;  // 1.5 * 2^52
    const double t = __fma_rn(x, 23.083120654223414, kMagic);
    const double Nd = __dsub_rn(t, kMagic);
    const int N = __double2loint(t);
    double r = __fma_rn(Nd, -0.04332169877307024, x);
    r = __fma_rn(Nd, -1.1926343307941173e-11, r);
    double p = -1.98412698412698412698e-04;  // (-1)^7 / 7!
    p = __fma_rn(p, r, 1.38888888888888888889e-03);
    p = __fma_rn(p, r, -8.33333333333333333333e-03);
    p = __fma_rn(p, r, 4.16666666666666666667e-02);
    p = __fma_rn(p, r, -1.66666666666666666667e-01);
    p = __fma_rn(p, r, 0.5);
    p = __fma_rn(p, r, -1.0);
    p = __fma_rn(p, r, 1.0);
    const double tb = tab[N & 15];
    const int q = min(N >> 4, 1010);
    const double sc = __hiloint2double(__double2hiint(tb) - (q << 20), __double2loint(tb));
    return __dmul_rn(p, sc);
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
    __shared__ double s_tab[16];
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
    double hmax = 0.0, hmin = INFINITY;
#pragma unroll
    for (int q = 0; q < kGB; q++) {
        const double h = __ldg(hg + min(b0 + q, m - 1));
        hmax = fmax(hmax, h);
        hmin = fmin(hmin, h);
        c[q] = 0.5 / (h * h);
        num[q] = 0.0;
        den[q] = 0.0;
    }
    // cap of t = d^2 - dmin^2 keeping every x = t c <= 9e7 (exp_neg_tab's
    // range: N = 16 x / ln2 must fit an int); a capped column still has
    // x >= 9e7 hmin^2/hmax^2 >= 700 for every bandwidth of the chunk when
    // hmax/hmin <= 300, so its weight stays ~1e-304.  Chunks spanning a wider
    // bandwidth ratio (extreme grids) clamp x per bandwidth instead (slow
    // path, block-uniform branch).
    const bool wide = hmax > 300.0 * hmin;
    const double ttcap = wide ? INFINITY : 1.8e8 * hmin * hmin;
    // column range that can matter for any row of the tile and bandwidth of
    // the chunk
    if (t < 16) s_tab[t] = kExp2Tab[t];
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
            // leave-one-out (Eq.(2) l != i): the row itself gets t = ttcap, i.e.
            // weight ~1e-304 next to the nearest neighbour's 1 -- below half
            // an ulp of every sum it joins, so the sums are unchanged
            const double tt = q == self ? ttcap : fmin(__fma_rn(d, d, -dmin2), ttcap);
            if (!wide) {
#pragma unroll
                for (int k = 0; k < kGB; k++) {
                    const double wgt = exp_neg_tab(tt * c[k], s_tab);
                    num[k] = __fma_rn(wgt, v.y, num[k]);
                    den[k] += wgt;
                }
            } else {
#pragma unroll
                for (int k = 0; k < kGB; k++) {
                    const double wgt = exp_neg_tab(fmin(tt * c[k], 1e4), s_tab);
                    num[k] = __fma_rn(wgt, v.y, num[k]);
                    den[k] += wgt;
                }
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
