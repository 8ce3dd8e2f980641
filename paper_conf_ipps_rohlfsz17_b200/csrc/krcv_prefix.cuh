// krcv_prefix.cuh -- the window-prefix path ("a
// sub-quadratic window-prefix variant").
//
// Same quantities as the per-pair sweep (krcv_sweep.cuh): for every sorted
// row r and every bandwidth h_b of the ascending grid, the window
// W_r(h_b) = { l != r : |x_l - x_r| < h_b } (<= for uniform; reading Q1),
// the running sums c, sum y, sum d^2, sum y d^2 over it (reading Q3), the LOO
// estimate Eq.(2), M (Q6) and the squared error of Eq.(1).
//
// What changes is how the running sums reach h_b.  The paper (§III
// P@14010-14984, §IV.B P@21724-22104) carries them from h_{b-1} and adds the
// additional neighbours one by one.  On the globally sorted array the window
// of row r is the index range (L_r(b), R_r(b)) minus r itself, so:
//   * the boundaries are found by a galloping search with the exact binary64
//     membership predicate (monotone along the sorted array), starting from
//     the previous bandwidth's boundaries -- window membership is identical to
//     the sweep's and the oracle's, bit for bit;
//   * the "additional values" of every bandwidth step are summed in O(1) as a
//     difference of prefix sums P[R] - P[L+1] of the moments
//     y, u, u^2, y u, y u^2 (u = x - o, o = the median x), kept in
//     double-double so the difference and the shift to the row's own origin,
//         sum (x_l - x_r)^2     = Suu  - delta (2 Su  - c' delta)
//         sum y_l (x_l - x_r)^2 = Syuu - delta (2 Syu - delta Sy)
//     (delta = x_r - o, c' = R - L - 1 including row r, whose own terms are
//     0 in both), lose nothing to cancellation (krcv_dd.cuh);
//   * sum y excludes row r by subtracting y_r (LOO, Eq.(2) l != i, Q8).
// Per (row, bandwidth) the work is O(log growth) + O(1); nothing is O(n) per
// row, so a grid search costs O(n m log) instead of O(n^2).
//
// Kernels:
//   pfx_tile_reduce_kernel  per tile of 256 ITEMS sorted records: moment terms
//                           and their dd totals
//   pfx_tile_scan_kernel    per tile: its offset (fixed-order sum of the
//                           earlier tiles' totals), prefix values P[k][0..n]
//                           and the plain
//                           sorted-x array xs[] (+-inf sentinels) the
//                           searches read
//   window_kernel<K>   a warp owns 32 consecutive sorted rows (one per lane),
//                      walks b = 0..m-1, emits (M e^2, M) per (tile, b) into
//                      the same tile-partial layout the sweep uses (a5).
#pragma once

#include "krcv_pdl.cuh"

#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

#include "krcv.h"
#include "krcv_dd.cuh"
#include "krcv_sweep.cuh"

namespace krcv {

constexpr int kPfxThreads = 256;      // prefix build CTA
constexpr int kPfxMoments = 8;        // slots reserved in the workspace (local-linear uses all 8)
constexpr int kWinWarps = 4;
constexpr int kWinThreads = kWinWarps * 32;
constexpr int kWinTasksPerSM = 256;   // warp tasks per SM the b-split aims for (measured: C3 nbc 7 -> 28, -9 %)
constexpr int kWinMinBper = 8;        // >= this many bandwidths per task
// Density statistic for the bucket table (krcv_window.cuh): the smallest
// x-distance spanned by kGapSpan + 1 consecutive sorted records, stored as
// the complement of its bit pattern (non-negative doubles order like their
// bits, so the complement orders inversely and atomicMax keeps the minimum;
// the status memset's 0 is below every stored value).
constexpr int kGapSpan = 64;

__device__ __forceinline__ void gap_stat(const double2 *__restrict__ xy, int n, int j, double &gmin)
{
    if (j + kGapSpan < n) gmin = fmin(gmin, xy[j + kGapSpan].x - xy[j].x);
}

__device__ __forceinline__ void gap_publish(double gmin, unsigned long long *__restrict__ gap_bits)
{
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) gmin = fmin(gmin, __shfl_xor_sync(0xffffffffu, gmin, d));
    if ((threadIdx.x & 31) == 0 && gmin < INFINITY)
        atomicMax(gap_bits, ~(unsigned long long)__double_as_longlong(fmax(gmin, 0.0)));
}

// Moments per kernel (slot order).  Epanechnikov: y, u, u^2, y u, y u^2.
// Triangular: y, u, y u.  Uniform: y.
// Pseudo-kernel id of the KDE moment set (krcv_kde.cuh): u, u^2, ..., u^5.
constexpr int kKdeMoments = 100;
// Pseudo-kernel id of the local-linear moment set (krcv_ll.cuh):
// y, u, u^2, u^3, u^4, y u, y u^2, y u^3.
constexpr int kLLMoments = 101;

template <int KERN>
struct NMom {
    static constexpr int v =
        KERN == kLLMoments ? 8 : (KERN == KR_UNIFORM ? 1 : (KERN == KR_TRIANGULAR ? 3 : 5));
};

template <int KERN>
__device__ __forceinline__ void moment_terms(double x, double y, double o, dd (&t)[kPfxMoments])
{
    if (KERN == kKdeMoments) {  // KDE: powers of u = x - o (y unused)
        const dd u = two_sum(x, -o);
        t[0] = u;
        t[1] = dd_mul(u, u);
        t[2] = dd_mul(t[1], u);
        t[3] = dd_mul(t[1], t[1]);
        t[4] = dd_mul(t[3], u);
        return;
    }
    if (KERN == kLLMoments) {  // local-linear: y, u .. u^4, y u .. y u^3
        const dd u = two_sum(x, -o);
        const dd u2 = dd_mul(u, u), u3 = dd_mul(u2, u);
        t[0] = dd_make(y);
        t[1] = u;
        t[2] = u2;
        t[3] = u3;
        t[4] = dd_mul(u2, u2);
        t[5] = dd_mul_d(u, y);
        t[6] = dd_mul_d(u2, y);
        t[7] = dd_mul_d(u3, y);
        return;
    }
    t[0] = dd_make(y);
    if (KERN != KR_UNIFORM) {
        const dd u = two_sum(x, -o);  // exact: u.hi + u.lo == x - o
        if (KERN == KR_EPANECHNIKOV) {
            const dd uu = dd_mul(u, u);
            t[1] = u;
            t[2] = uu;
            t[3] = dd_mul_d(u, y);
            t[4] = dd_mul_d(uu, y);
        } else {
            t[1] = u;
            t[2] = dd_mul_d(u, y);
        }
    }
}

// Prefix storage.  Nadaraya-Watson moment sets (uniform / Epanechnikov /
// triangular) are stored in blocks of kRecBlock indices, each block holding
// the block's values plane after plane: Epanechnikov planes (y, u) and
// (u^2, y u) of 16-byte pairs and (y u^2) of doubles -- 40 bytes per index;
// triangular (y, u) and (y u); uniform (y).  Moment slot k of index j is at
// double offset  (j / kRecBlock) BS + plane_off(k) + (j % kRecBlock) w(k) + sub(k).
// A warp whose 32 lanes read 32 consecutive indices loads 512 contiguous
// bytes per pair plane (4 L1 wavefronts; an array of 40-byte structures would
// span 10 lines per load), and the planes of one index are a fixed 16 / 32 KB
// apart: immediate offsets of one address.  The lo words follow the hi words
// at double offset pk_lo_off(ps).  (No padding: the whole C4 working set --
// hi records, sorted x, bucket table -- must stay inside the 126 MB L2;
// profiles/r02f_* measured 12-15 GB of DRAM reads per launch when it did not.)
// The KDE and local-linear sets keep structure-of-arrays planes (hi of moment
// k at P + 2k ps, lo at P + (2k+1) ps).
constexpr int kRecBlock = 1024;
// KRCV_REC_AOS=1 (build time, A/B runs): records as an array of structures of
// S + 1 doubles (the moments, then the index j as a double) instead of the
// blocked planes.
#ifndef KRCV_REC_AOS
#define KRCV_REC_AOS 0
#endif
constexpr bool kRecAos = KRCV_REC_AOS != 0;

template <int KERN>
struct PfxRec {
    static constexpr int S0 = KERN == KR_EPANECHNIKOV ? 5 : (KERN == KR_TRIANGULAR ? 3 : (KERN == KR_UNIFORM ? 1 : 0));
    static constexpr int S = (kRecAos && S0) ? S0 + 1 : S0;  // doubles per index (AoS: + the index slot)
    static constexpr int BS = S * kRecBlock;  // doubles per block (all planes)
    // plane of slot k: width 2 for slots 0..2*(S/2)-1, width 1 for the odd last slot
    static __host__ __device__ constexpr int width(int k) { return k < 2 * (S / 2) ? 2 : 1; }
    static __host__ __device__ constexpr int plane_off(int k) { return (k / 2) * 2 * kRecBlock; }
    static __host__ __device__ constexpr int sub(int k) { return k < 2 * (S / 2) ? (k & 1) : 0; }
};

// index slots reserved for prefix stride ps (>= n + 1): whole blocks
__host__ __device__ __forceinline__ size_t pk_slots(int ps)
{
    return ((size_t)ps + kRecBlock - 1) / kRecBlock * kRecBlock;
}

// doubles of one (hi or lo) record array for prefix stride ps
template <int KERN>
__host__ __device__ __forceinline__ size_t pk_lo_off(int ps)
{
    return (size_t)PfxRec<KERN>::S * pk_slots(ps);
}

// double offset of moment slot k of index j (j >= 0): one shift and one
// 32 x 32 -> 64-bit multiply-add plus constants
template <int KERN>
__device__ __forceinline__ size_t pk_off(int k, int j)
{
    using R = PfxRec<KERN>;
    if (kRecAos) return (size_t)j * R::S + k;
    const unsigned u = (unsigned)j;
    return (size_t)(u >> 10) * (unsigned)R::BS +
           (size_t)((u & (kRecBlock - 1)) * (unsigned)R::width(k) + (unsigned)(R::plane_off(k) + R::sub(k)));
}

template <int KERN>
__device__ __forceinline__ void pk_store(double *__restrict__ P, int ps, int k, int j, dd v)
{
    if (PfxRec<KERN>::S) {
        P[pk_off<KERN>(k, j)] = v.hi;
        P[pk_lo_off<KERN>(ps) + pk_off<KERN>(k, j)] = v.lo;
    } else {
        P[(size_t)(2 * k) * ps + j] = v.hi;
        P[(size_t)(2 * k + 1) * ps + j] = v.lo;
    }
}

// the AoS layout's index slot (the blocked layout has none)
template <int KERN>
__device__ __forceinline__ void pk_store_index(double *__restrict__ P, int ps, int j)
{
    constexpr int S = PfxRec<KERN>::S;
    if (kRecAos && S) {
        P[(size_t)j * S + S - 1] = (double)j;
        P[pk_lo_off<KERN>(ps) + (size_t)j * S + S - 1] = 0.0;
    }
}

template <int KERN>
__device__ __forceinline__ double pk_hi(const double *__restrict__ P, int ps, int k, int j)
{
    return PfxRec<KERN>::S ? P[pk_off<KERN>(k, j)] : P[(size_t)(2 * k) * ps + j];
}

template <int KERN>
__device__ __forceinline__ dd pk_dd(const double *__restrict__ P, int ps, int k, int j)
{
    return PfxRec<KERN>::S ? dd{P[pk_off<KERN>(k, j)], P[pk_lo_off<KERN>(ps) + pk_off<KERN>(k, j)]}
                           : dd{P[(size_t)(2 * k) * ps + j], P[(size_t)(2 * k + 1) * ps + j]};
}

template <int KERN>
__device__ __forceinline__ dd pk_wsum(const double *__restrict__ P, int ps, int k, int a, int b)
{
    return dd_sub(pk_dd<KERN>(P, ps, k, b), pk_dd<KERN>(P, ps, k, a));
}

__device__ __forceinline__ dd ld_dd(const double2 *p) { const double2 v = *p; return dd{v.x, v.y}; }
__device__ __forceinline__ void st_dd(double2 *p, dd v) { *p = make_double2(v.hi, v.lo); }

// origin o: the median record of the sorted array (keeps |u| small).
__device__ __forceinline__ double pfx_origin(const double2 *xy, int n) { return xy[n >> 1].x; }

// First gallop step of a chunk's cold search at bandwidth h: half the
// window size a uniform density would give, (n - 1) h / (x_max - x_min) / 2
// (>= 1).  Chunks after the first start far from the row, and a gallop from
// step 1 would spend ~2 log2(window) probes per side getting there; any step
// keeps the search exact (the gallop / bisection verify every boundary).
__device__ __forceinline__ int cold_step(const double *__restrict__ xs, int n, double h)
{
    const double span = xs[n - 1] - xs[0];
    if (!(span > 0.0)) return 1;
    const double e = 0.5 * (double)(n - 1) * (h / span);
    return e >= (double)n ? n : (e < 1.0 ? 1 : (int)e);
}

// ---------------------------------------------------------------- build
// Two-phase fixed-order scan (bit-reproducible; a decoupled look-back
// would make the dd rounding depend on timing): tile totals, then every tile
// sums its predecessors' totals itself and scans its records.  A tile is
// 256 ITEMS sorted records; thread t of its CTA owns records ITEMS t ..
// ITEMS t + ITEMS - 1 of the tile.  ITEMS = 4 (tile 1,024) for large n, 1
// (tile 256) for small n so that the scan spreads over more CTAs
// (pfx_items() in krcv_device.cu).
constexpr int kPfxItemsMax = 4;
constexpr int kPfxTileMin = kPfxThreads;  // the workspace sizes tile totals for this

__device__ __forceinline__ dd shfl_up_dd(dd v, int d)
{
    return dd{__shfl_up_sync(0xffffffffu, v.hi, d), __shfl_up_sync(0xffffffffu, v.lo, d)};
}

__device__ __forceinline__ dd shfl_xor_dd(dd v, int d)
{
    return dd{__shfl_xor_sync(0xffffffffu, v.hi, d), __shfl_xor_sync(0xffffffffu, v.lo, d)};
}

template <int KERN, int ITEMS, bool GAP>
__device__ __forceinline__ void pfx_reduce_body(const double2 *__restrict__ xy, int n, double2 *__restrict__ tot,
                                                int ntiles, unsigned long long *__restrict__ ymax_bits,
                                                unsigned long long *__restrict__ gap_bits, int tile);
template <int KERN, int ITEMS, bool GAP, bool CG>
__device__ __forceinline__ void pfx_scan_body(const double2 *__restrict__ xy, int n, const double2 *__restrict__ tot,
                                              int ntiles, double *__restrict__ P, int pstride,
                                              double *__restrict__ xs, unsigned long long *__restrict__ gap_bits,
                                              int tile);

// Phase 1: per-tile totals of the moment terms -> tot[k][tile].
template <int KERN, int ITEMS>
__global__ void __launch_bounds__(kPfxThreads)
pfx_tile_reduce_kernel(const double2 *__restrict__ xy, int n, double2 *__restrict__ tot, int ntiles,
                       unsigned long long *__restrict__ ymax_bits)
{
    pdl_wait();  // krcv_pdl.cuh
    pfx_reduce_body<KERN, ITEMS, false>(xy, n, tot, ntiles, ymax_bits, nullptr, blockIdx.x);
}

// Phase 1 body (also used by the fused build, krcv_window.cuh): tile `tile`'s
// dd totals -> tot[k][tile], max|y|, and with GAP the density statistic.
template <int KERN, int ITEMS, bool GAP>
__device__ __forceinline__ void pfx_reduce_body(const double2 *__restrict__ xy, int n, double2 *__restrict__ tot,
                                                int ntiles, unsigned long long *__restrict__ ymax_bits,
                                                unsigned long long *__restrict__ gap_bits, int tile)
{
    constexpr int K = NMom<KERN>::v;
    __shared__ double2 wsum[K][kPfxThreads / 32];
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int j0 = tile * (kPfxThreads * ITEMS) + t * ITEMS;
    const double o = pfx_origin(xy, n);
    dd acc[kPfxMoments];
#pragma unroll
    for (int k = 0; k < K; k++) acc[k] = dd{0.0, 0.0};
    double ym = 0.0, gmin = INFINITY;
#pragma unroll
    for (int q = 0; q < ITEMS; q++) {
        if (j0 + q < n) {
            const double2 v = xy[j0 + q];
            ym = fmax(ym, fabs(v.y));
            if (GAP && PfxRec<KERN>::S) gap_stat(xy, n, j0 + q, gmin);
            dd tm[kPfxMoments];
            moment_terms<KERN>(v.x, v.y, o, tm);
#pragma unroll
            for (int k = 0; k < K; k++) acc[k] = dd_add(acc[k], tm[k]);
        }
    }
#pragma unroll
    for (int k = 0; k < K; k++) {
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) acc[k] = dd_add(acc[k], shfl_xor_dd(acc[k], d));
        if (lane == 0) st_dd(&wsum[k][w], acc[k]);
    }
    // max |y| over all records (the window kernel's fast-path bound);
    // non-negative doubles order like their bit patterns
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) ym = fmax(ym, __shfl_xor_sync(0xffffffffu, ym, d));
    if (lane == 0 && ym > 0.0) atomicMax(ymax_bits, (unsigned long long)__double_as_longlong(ym));
    if (GAP && PfxRec<KERN>::S) gap_publish(gmin, gap_bits);
    __syncthreads();
    if (t < K) {
        dd a = dd{0.0, 0.0};
        for (int q = 0; q < kPfxThreads / 32; q++) a = dd_add(a, ld_dd(&wsum[t][q]));
        st_dd(tot + (size_t)t * ntiles + tile, a);
    }
}

// Phase 3: in-tile exclusive scan + tile offset -> P[k][j] = sum_{l<j} t_k(l)
// for j in the tile (and P[k][n] by the last tile), plus the plain sorted-x
// array xs (with -inf / +inf sentinels) used by the window searches.
template <int KERN, int ITEMS>
__global__ void __launch_bounds__(kPfxThreads)
pfx_tile_scan_kernel(const double2 *__restrict__ xy, int n, const double2 *__restrict__ tot, int ntiles,
                     double *__restrict__ P, int pstride, double *__restrict__ xs,
                     unsigned long long *__restrict__ gap_bits)
{
    pdl_wait();  // krcv_pdl.cuh
    pfx_scan_body<KERN, ITEMS, true, false>(xy, n, tot, ntiles, P, pstride, xs, gap_bits, blockIdx.x);
}

// Phase 3 body (also used by the fused build): tile `tile`'s offset, scan,
// records and xs; GAP: the density statistic here; CG: read the other tiles'
// totals through L2 (they were written in this same launch).
template <int KERN, int ITEMS, bool GAP, bool CG>
__device__ __forceinline__ void pfx_scan_body(const double2 *__restrict__ xy, int n, const double2 *__restrict__ tot,
                                              int ntiles, double *__restrict__ P, int pstride,
                                              double *__restrict__ xs, unsigned long long *__restrict__ gap_bits,
                                              int tile)
{
    constexpr int K = NMom<KERN>::v;
    __shared__ double2 wsum[K][kPfxThreads / 32];
    __shared__ double2 base_s[K];
    // this tile's offset: the totals of all earlier tiles, summed in a fixed
    // order (strided per thread, then a fixed tree) -- no separate scan launch
    {
        const int t = threadIdx.x, lane = t & 31, w = t >> 5;
        dd a[kPfxMoments];
#pragma unroll
        for (int k = 0; k < K; k++) {
            a[k] = dd{0.0, 0.0};
            for (int q = t; q < tile; q += kPfxThreads) {
                const double2 *pq = tot + (size_t)k * ntiles + q;
                a[k] = dd_add(a[k], CG ? dd{__ldcg(&pq->x), __ldcg(&pq->y)} : ld_dd(pq));
            }
#pragma unroll
            for (int d = 16; d > 0; d >>= 1) a[k] = dd_add(a[k], shfl_xor_dd(a[k], d));
            if (lane == 0) st_dd(&wsum[k][w], a[k]);
        }
        __syncthreads();
        if (t < K) {
            dd b = dd{0.0, 0.0};
            for (int q = 0; q < kPfxThreads / 32; q++) b = dd_add(b, ld_dd(&wsum[t][q]));
            st_dd(&base_s[t], b);
        }
        __syncthreads();
    }
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int j0 = tile * (kPfxThreads * ITEMS) + t * ITEMS;
    if (tile == 0 && t < kPad) {
        xs[-1 - t] = -INFINITY;
        xs[n + t] = INFINITY;
    }
    const double o = pfx_origin(xy, n);
    // ITEMS > 1: the tile's records staged through shared memory (coalesced
    // loads and xs stores; each thread then reads its ITEMS consecutive
    // records), and the moment terms recomputed for the record stores instead
    // of held in registers across the scan (124 -> fewer registers: the
    // kernel is latency-bound at 2 CTAs per SM otherwise, profiles/r02/r02ab_*)
    __shared__ double2 sxy[ITEMS > 1 ? kPfxThreads * ITEMS : 1];
    if (ITEMS > 1) {
        const int tb = tile * (kPfxThreads * ITEMS);
#pragma unroll
        for (int q = 0; q < ITEMS; q++) {
            const int jj = tb + q * kPfxThreads + t;
            const double2 v = jj < n ? xy[jj] : make_double2(0.0, 0.0);
            sxy[q * kPfxThreads + t] = v;
            if (jj < n) xs[jj] = v.x;
        }
        __syncthreads();
    }
    auto rec = [&](int q) { return ITEMS > 1 ? sxy[t * ITEMS + q] : xy[j0 + q]; };
    dd tm[ITEMS > 1 ? 1 : ITEMS][kPfxMoments];
    dd acc[kPfxMoments];
    double gmin = INFINITY;
#pragma unroll
    for (int k = 0; k < K; k++) acc[k] = dd{0.0, 0.0};
#pragma unroll
    for (int q = 0; q < ITEMS; q++) {
        dd (&tq)[kPfxMoments] = tm[ITEMS > 1 ? 0 : q];
        if (j0 + q < n) {
            const double2 v = rec(q);
            if (ITEMS == 1) xs[j0 + q] = v.x;
            if (GAP && PfxRec<KERN>::S) gap_stat(xy, n, j0 + q, gmin);
            moment_terms<KERN>(v.x, v.y, o, tq);
        } else {
#pragma unroll
            for (int k = 0; k < K; k++) tq[k] = dd{0.0, 0.0};
        }
#pragma unroll
        for (int k = 0; k < K; k++) acc[k] = dd_add(acc[k], tq[k]);
    }
    if (GAP && PfxRec<KERN>::S) gap_publish(gmin, gap_bits);
    // exclusive scan of the thread totals across the CTA
    dd ex[kPfxMoments];
#pragma unroll
    for (int k = 0; k < K; k++) {
        dd inc = acc[k];
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const dd u = shfl_up_dd(inc, d);
            if (lane >= d) inc = dd_add(u, inc);
        }
        if (lane == 31) st_dd(&wsum[k][w], inc);
        const dd u = shfl_up_dd(inc, 1);
        ex[k] = lane == 0 ? dd{0.0, 0.0} : u;
    }
    __syncthreads();
    if (ITEMS == 1) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            dd base = ld_dd(&base_s[k]);
            for (int q = 0; q < w; q++) base = dd_add(base, ld_dd(&wsum[k][q]));
            const dd run = dd_add(base, ex[k]);
            if (j0 <= n) {
                pk_store<KERN>(P, pstride, k, j0, run);
                if (k == 0) pk_store_index<KERN>(P, pstride, j0);
            }
        }
        return;
    }
    dd run[kPfxMoments];
#pragma unroll
    for (int k = 0; k < K; k++) {
        dd base = ld_dd(&base_s[k]);
        for (int q = 0; q < w; q++) base = dd_add(base, ld_dd(&wsum[k][q]));
        run[k] = dd_add(base, ex[k]);
    }
#pragma unroll
    for (int q = 0; q < ITEMS; q++) {
        if (j0 + q > n) break;
#pragma unroll
        for (int k = 0; k < K; k++) pk_store<KERN>(P, pstride, k, j0 + q, run[k]);
        pk_store_index<KERN>(P, pstride, j0 + q);
        if (q + 1 < ITEMS && j0 + q < n) {  // the same terms as the first pass (deterministic)
            const double2 v = rec(q);
            dd tq[kPfxMoments];
            moment_terms<KERN>(v.x, v.y, o, tq);
#pragma unroll
            for (int k = 0; k < K; k++) run[k] = dd_add(run[k], tq[k]);
        }
    }
}

// One-CTA build for small n (a single launch instead of two; the two-phase
// build is latency-bound there).  Thread t owns the contiguous records
// [t I, t I + I), I = ceil(n / kPfx1Threads): pass 1 sums its terms in order,
// a fixed-order block scan (warp shuffles, then warp 0 over the warp totals)
// gives each thread its exclusive offset, pass 2 recomputes the terms and
// writes the running prefix P[k][j] (j = 0 .. n), xs and the sentinels.
// Every sum is in a fixed order: bit-reproducible, like the two-phase build
// (whose different order rounds differently in the last dd bits).
constexpr int kPfx1Threads = 512;

template <int KERN>
__global__ void __launch_bounds__(kPfx1Threads)
pfx_one_cta_kernel(const double2 *__restrict__ xy, int n, double *__restrict__ P, int pstride,
                   double *__restrict__ xs, unsigned long long *__restrict__ ymax_bits,
                   unsigned long long *__restrict__ gap_bits)
{
    constexpr int K = NMom<KERN>::v;
    constexpr int W = kPfx1Threads / 32;
    __shared__ double2 wtot[K][W];
    __shared__ double2 woff[K][W];
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int I = (n + kPfx1Threads - 1) / kPfx1Threads;
    const int j0 = min(n, t * I), j1 = min(n, j0 + I);
    const double o = pfx_origin(xy, n);
    if (t < kPad) {
        xs[-1 - t] = -INFINITY;
        xs[n + t] = INFINITY;
    }
    // pass 1: this thread's totals
    dd acc[kPfxMoments];
#pragma unroll
    for (int k = 0; k < K; k++) acc[k] = dd{0.0, 0.0};
    double ym = 0.0, gmin = INFINITY;
    for (int j = j0; j < j1; j++) {
        const double2 v = xy[j];
        ym = fmax(ym, fabs(v.y));
        if (PfxRec<KERN>::S) gap_stat(xy, n, j, gmin);
        dd tm[kPfxMoments];
        moment_terms<KERN>(v.x, v.y, o, tm);
#pragma unroll
        for (int k = 0; k < K; k++) acc[k] = dd_add(acc[k], tm[k]);
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) ym = fmax(ym, __shfl_xor_sync(0xffffffffu, ym, d));
    if (lane == 0 && ym > 0.0) atomicMax(ymax_bits, (unsigned long long)__double_as_longlong(ym));
    if (PfxRec<KERN>::S) gap_publish(gmin, gap_bits);
    // exclusive scan of the thread totals: within the warp, then over the warps
    dd ex[kPfxMoments];
#pragma unroll
    for (int k = 0; k < K; k++) {
        dd inc = acc[k];
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const dd u = shfl_up_dd(inc, d);
            if (lane >= d) inc = dd_add(u, inc);
        }
        if (lane == 31) st_dd(&wtot[k][w], inc);
        const dd u = shfl_up_dd(inc, 1);
        ex[k] = lane == 0 ? dd{0.0, 0.0} : u;
    }
    __syncthreads();
    if (w == 0) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            dd inc = lane < W ? ld_dd(&wtot[k][lane]) : dd{0.0, 0.0};
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const dd u = shfl_up_dd(inc, d);
                if (lane >= d) inc = dd_add(u, inc);
            }
            const dd u = shfl_up_dd(inc, 1);
            if (lane < W) st_dd(&woff[k][lane], lane == 0 ? dd{0.0, 0.0} : u);
        }
    }
    __syncthreads();
    // pass 2: running prefix over this thread's records
    dd run[kPfxMoments];
#pragma unroll
    for (int k = 0; k < K; k++) run[k] = dd_add(ld_dd(&woff[k][w]), ex[k]);
    for (int j = j0; j < j1; j++) {
        const double2 v = xy[j];
        xs[j] = v.x;
        dd tm[kPfxMoments];
        moment_terms<KERN>(v.x, v.y, o, tm);
#pragma unroll
        for (int k = 0; k < K; k++) {
            pk_store<KERN>(P, pstride, k, j, run[k]);
            run[k] = dd_add(run[k], tm[k]);
        }
        pk_store_index<KERN>(P, pstride, j);
    }
    if (j1 == n && j0 < n) {  // the thread holding the last record writes P[k][n]
#pragma unroll
        for (int k = 0; k < K; k++) pk_store<KERN>(P, pstride, k, n, run[k]);
        pk_store_index<KERN>(P, pstride, n);
    }
}

// ---------------------------------------------------------------- windows
// New boundaries for bandwidth h from the previous ones, in offsets from the
// row: the right side probes xs[r + k], the left side xs[r - k]; "inside" is
// the exact binary64 predicate of reading Q1 and is monotone in k.  On entry
// every offset in (0, kR) / (0, kL) is inside (the previous windows); on exit
// kR / kL are the first offsets outside.  xs carries +-inf sentinels, so
// offset n - r (right) and r + 1 (left) are outside every window.
// Gallop (first step = the previous growth gR / gL, then doubling) and
// bisect; both sides advance in the same loop iteration (memory-level
// parallelism).  (Predicted-bracket and interpolation variants issued more
// instructions than they saved probes: profiles/r01f_*, r01l_*.)
template <int KERN>
__device__ __forceinline__ void window_bounds(const double *__restrict__ xs, int n, int r, double xr, double h,
                                              int &kR, int &kL, int gR, int gL)
{
    // the row's base pointer, laundered through an empty asm so the compiler
    // keeps it in a register instead of re-deriving xs + (r + k) in 64-bit
    // arithmetic at every probe (4 instructions -> 1 IMAD.WIDE)
    unsigned long long base = reinterpret_cast<unsigned long long>(xs + r);
    asm("" : "+l"(base));
    const double *__restrict__ xsr = reinterpret_cast<const double *>(base);
    int rlo = kR - 1, rhi = 0, rstep = gR;  // rlo: inside (or the row itself)
    int llo = kL - 1, lhi = 0, lstep = gL;
    const int kRmax = n - r, kLmax = r + 1;
    int rg = 1, lg = 1;  // int flags: bools cost byte-permute instructions here
    // Predicted bracket: the boundary is expected about one growth g beyond
    // the previous one, give or take a few sqrt(g) (Poisson spread of the
    // points added).  Probe g - s and g + s (s = 3 sqrt(g)) on both sides at
    // once -- four independent loads -- and bisect the bracket that holds
    // the boundary; if both probes are inside, keep galloping from g + s.
    // Any outcome leaves a valid state for the loops below (exactness does
    // not depend on the prediction).
    if (gR >= 4) {
        const int sR = (int)(3.0f * sqrtf((float)gR));
        const int p1 = min(rlo + max(1, gR - sR), kRmax), p2 = min(rlo + gR + sR, kRmax);
        const int in1 = inside<KERN>(__ldg(xsr + p1) - xr, h), in2 = inside<KERN>(__ldg(xsr + p2) - xr, h);
        rhi = !in1 ? p1 : (!in2 ? p2 : 0);
        rlo = !in1 ? rlo : (!in2 ? p1 : p2);
        rstep = 2 * sR + 1;
        rg = in1 & in2;
    }
    if (gL >= 4) {
        const int sL = (int)(3.0f * sqrtf((float)gL));
        const int p1 = min(llo + max(1, gL - sL), kLmax), p2 = min(llo + gL + sL, kLmax);
        const int in1 = inside<KERN>(xr - __ldg(xsr - p1), h), in2 = inside<KERN>(xr - __ldg(xsr - p2), h);
        lhi = !in1 ? p1 : (!in2 ? p2 : 0);
        llo = !in1 ? llo : (!in2 ? p1 : p2);
        lstep = 2 * sL + 1;
        lg = in1 & in2;
    }
    while (rg | lg) {
        if (rg) {
            const int k = min(rlo + rstep, kRmax);
            const int in = inside<KERN>(__ldg(xsr + k) - xr, h);
            rlo = in ? k : rlo;
            rhi = in ? rhi : k;
            rstep <<= in;
            rg = in;
        }
        if (lg) {
            const int k = min(llo + lstep, kLmax);
            const int in = inside<KERN>(xr - __ldg(xsr - k), h);
            llo = in ? k : llo;
            lhi = in ? lhi : k;
            lstep <<= in;
            lg = in;
        }
    }
    while (rhi - rlo > 1 || lhi - llo > 1) {
        if (rhi - rlo > 1) {
            const int k = (rlo + rhi) >> 1;
            if (inside<KERN>(__ldg(xsr + k) - xr, h)) rlo = k; else rhi = k;
        }
        if (lhi - llo > 1) {
            const int k = (llo + lhi) >> 1;
            if (inside<KERN>(xr - __ldg(xsr - k), h)) llo = k; else lhi = k;
        }
    }
    kR = rhi;
    kL = lhi;
}

// Prefix storage: structure of arrays, moment k's hi parts at
// P + 2k pstride, lo parts at P + (2k+1) pstride (the fast path below reads
// only the hi words).
__device__ __forceinline__ double ld_hi(const double *__restrict__ P, int ps, int k, int j)
{
    return P[(size_t)(2 * k) * ps + j];
}

__device__ __forceinline__ dd ld_pdd(const double *__restrict__ P, int ps, int k, int j)
{
    return dd{P[(size_t)(2 * k) * ps + j], P[(size_t)(2 * k + 1) * ps + j]};
}

// Window sums of moment k over sorted indices [a, b): P[b] - P[a], in dd.
__device__ __forceinline__ dd wsum(const double *__restrict__ P, int ps, int k, int a, int b)
{
    return dd_sub(ld_pdd(P, ps, k, b), ld_pdd(P, ps, k, a));
}

// Fast-path acceptance.  The hi words are the prefix sums
// rounded to nearest, so a difference of two of them carries an absolute
// error <= eps/2 (|P[b]| + |P[a]|) + eps |diff|; the shift to the row adds
// errors of the order of the magnitudes it combines.  E1 / E2 / E0 bound
// those magnitudes for sum d^2, sum y d^2 and sum y; the fast result is
// kept only if kFastSlack eps times them is below kFastTol of the
// denominator (and, for the numerator, of den * max|y|), which bounds the
// fast path's relative error in den and its absolute error in g_{-i} by
// kFastTol (times max|y|).  Otherwise the window is recomputed in dd.
// a / b for finite b != 0 with normal 1/b: hardware reciprocal estimate, two
// Newton steps and one residual correction -- within 1 ulp of the correctly
// rounded quotient, branch-free (IEEE division adds a slow-path test).
#ifndef KRCV_FASTDIV
#define KRCV_FASTDIV 1
#endif
__device__ __forceinline__ double fast_div(double a, double b)
{
    if (!KRCV_FASTDIV) return a / b;
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(b));
    double e = fma(-b, r, 1.0);
    r = fma(r, e, r);
    e = fma(-b, r, 1.0);
    r = fma(r, e, r);
    const double q = a * r;
    return fma(r, fma(-b, q, a), q);
}

#ifndef KRCV_EFACT
#define KRCV_EFACT 1  // factored fast-path bound (build-time A/B)
#endif
constexpr double kFastSlack = 16.0 * 0x1p-53;
constexpr double kFastTol = 0x1p-44;

// Per-row state of the window kernel.
struct WinRow {
    int r;       // sorted row index
    double xr, yr;
    dd del;      // x_r - o, exact
};

// The Epanechnikov fast path's anchored record set for a row (win_kernel,
// krcv_window.cuh): pa = the anchored copies (hi words, blocked layout, copy
// j at virtual indices j S + k), joff = j S for the row's anchor j, the row's
// shift dla = fl(x_r - o_j), and the global origin o (the dd path recomputes
// x_r - o from it).  Anchored words are within (eps/2 + 2^-57) of their
// magnitude of the exact anchored sums, or NaN (the fast test then fails and
// the window is recomputed from the global dd records).  Without it the fast
// path reads the global records about o with del.hi.
struct WinAnc {
    const double *pa;
    int joff;
    double dla, o;
};

// Squared LOO error of row `w` at bandwidth h with window [A, R) \ {r}
// (c = R - A - 1 >= 1): prefix differences (fast path or dd), Q14 guard,
// Eq.(2), Eq.(1)'s (y_r - g)^2.  Triangular needs P[r], P[r+1] (pr, pr1).
template <int KERN>
__device__ __forceinline__ double window_e2(const WinRow &w, int A, int R, int c, double h,
                                            const double2 *__restrict__ xy, const double *__restrict__ P, int ps,
                                            double ymax, const WinAnc *an = nullptr)
{
    const int r = w.r;
    const double xr = w.xr, yr = w.yr;
    const dd del = w.del;
    const double dl = del.hi, adl = fabs(del.hi);
    double g;
    if (KERN == KR_UNIFORM) {
        const double pb = pk_hi<KERN>(P, ps, 0, R), pa = pk_hi<KERN>(P, ps, 0, A);
        double sy = (pb - pa) - yr;
        if (!(kFastSlack * (fabs(pb) + fabs(pa) + fabs(yr)) <= kFastTol * (double)c * ymax))
            sy = dd_sub_to_d(pk_wsum<KERN>(P, ps, 0, A, R), dd_make(yr));
        g = fast_div(sy, (double)c);
    } else {
        const double hk = (KERN == KR_EPANECHNIKOV) ? h * h : h;
        double sy, s1, sy1, num, den;
        bool fast = false;
        if (KERN == KR_EPANECHNIKOV) {
            // fast path: hi words only, plain double (error test: see kFastTol)
            // records R and A (PfxRec planes (y, u), (u^2, y u), (y u^2)): two 16-byte and one
            // 8-byte load each, fixed offsets from one address
            const double *base = an ? an->pa : P;
            const int Rv = an ? R + an->joff : R, Av = an ? A + an->joff : A;  // virtual indices of copy j
            const double *pr = base + pk_off<KERN>(0, Rv);
            const double *pa = base + pk_off<KERN>(0, Av);
            const double dlf = an ? an->dla : dl, adlf = fabs(dlf);
            const int q2 = kRecAos ? 2 : 2 * kRecBlock;  // offset of the (u^2, y u) pair
            const double2 r01 = __ldg(reinterpret_cast<const double2 *>(pr));
            const double2 r23 = __ldg(reinterpret_cast<const double2 *>(pr + q2));
            const double2 a01 = __ldg(reinterpret_cast<const double2 *>(pa));
            const double2 a23 = __ldg(reinterpret_cast<const double2 *>(pa + q2));
            double yuu_b, yuu_a, c1;
            if (kRecAos) {  // (y u^2, j) pair: the count is a difference of loaded slots
                const double2 r45 = __ldg(reinterpret_cast<const double2 *>(pr + 4));
                const double2 a45 = __ldg(reinterpret_cast<const double2 *>(pa + 4));
                yuu_b = r45.x;
                yuu_a = a45.x;
                c1 = r45.y - a45.y;
            } else {
                yuu_b = __ldg(pr + 4 * kRecBlock - (int)((unsigned)Rv & (kRecBlock - 1)));
                yuu_a = __ldg(pa + 4 * kRecBlock - (int)((unsigned)Av & (kRecBlock - 1)));
                c1 = (double)(c + 1);  // range count R - A, row r included (its terms vanish)
            }
            const double y_b = r01.x, y_a = a01.x, u_b = r01.y, u_a = a01.y;
            const double uu_b = r23.x, uu_a = a23.x, yu_b = r23.y, yu_a = a23.y;
            const double Sy = y_b - y_a, Su = u_b - u_a, Suu = uu_b - uu_a;
            const double Syu = yu_b - yu_a, Syuu = yuu_b - yuu_a;
            s1 = fma(-dlf, fma(-c1, dlf, 2.0 * Su), Suu);
            sy1 = fma(-dlf, fma(-dlf, Sy, 2.0 * Syu), Syuu);
            sy = Sy - yr;
            num = fma(hk, sy, -sy1);
            den = fma(hk, c1 - 1.0, -s1);
            const double ay = fabs(y_b) + fabs(y_a);
            // E1 = |uu_b| + |uu_a| + 2|d| (|u_b| + |u_a|) + 2 c1 |d| (|d| + h),
            // E2 = |yuu_b| + |yuu_a| + 2|d| (|yu_b| + |yu_a|) + 2 d^2 ay + 2 c1 max|y| |d| (|d| + h),
            // factored (the same bounds to rounding, which the slack covers)
#if KRCV_EFACT
            const double dh = adlf + h, d2 = 2.0 * adlf;
            const double E1 = fma(d2, fma(c1, dh, fabs(u_b) + fabs(u_a)), fabs(uu_b) + fabs(uu_a));
            const double E2 = fma(d2, fma(c1 * ymax, dh, fma(adlf, ay, fabs(yu_b) + fabs(yu_a))),
                                  fabs(yuu_b) + fabs(yuu_a));
#else
            const double E1 = fabs(uu_b) + fabs(uu_a) + 2.0 * adlf * (fabs(u_b) + fabs(u_a)) +
                              2.0 * c1 * adlf * (adlf + h);
            const double E2 = fabs(yuu_b) + fabs(yuu_a) + 2.0 * adlf * (fabs(yu_b) + fabs(yu_a)) +
                              2.0 * adlf * adlf * ay + 2.0 * c1 * ymax * adlf * (adlf + h);
#endif
            const double E0 = ay + fabs(yr);
            // kFastSlack E1 <= kFastTol den, kFastSlack (hk E0 + E2) <= kFastTol den ymax, with the
            // exact power-of-two ratio kFastTol / kFastSlack folded in
            constexpr double kR = kFastTol / kFastSlack;
            fast = E1 <= kR * den && fma(hk, E0, E2) <= den * (kR * ymax);
        }
        if (!fast) {
            if (KERN == KR_EPANECHNIKOV) {
                // the records' hi and lo words at fixed offsets from two addresses
                const size_t lo = pk_lo_off<KERN>(ps);
                const double *pr = P + pk_off<KERN>(0, R), *pa = P + pk_off<KERN>(0, A);
                const int q2 = kRecAos ? 2 : 2 * kRecBlock;
                const int orr = kRecAos ? 4 : 4 * kRecBlock - (int)((unsigned)R & (kRecBlock - 1));
                const int oaa = kRecAos ? 4 : 4 * kRecBlock - (int)((unsigned)A & (kRecBlock - 1));
                auto wd = [&](int offr, int offa) {
                    return dd_sub(dd{pr[offr], pr[lo + offr]}, dd{pa[offa], pa[lo + offa]});
                };
                const dd Sy = wd(0, 0);
                const dd Su = wd(1, 1);
                const dd Suu = wd(q2, q2);
                const dd Syu = wd(q2 + 1, q2 + 1);
                const dd Syuu = wd(orr, oaa);
                const dd dlt = an ? two_sum(xr, -an->o) : del;  // x_r - o, exact (anchored rows keep none)
                const dd t1 = dd_sub(dd_twice(Su), dd_mul_d_raw(dlt, (double)(c + 1)));
                s1 = dd_sub_to_d(Suu, dd_mul_raw(dlt, t1));
                const dd t2 = dd_sub(dd_twice(Syu), dd_mul_raw(dlt, Sy));
                sy1 = dd_sub_to_d(Syuu, dd_mul_raw(dlt, t2));
                sy = dd_sub_to_d(Sy, dd_make(yr));
            } else {  // triangular: right (r, R) and left [A, r) separately
                const dd SyR = pk_wsum<KERN>(P, ps, 0, r + 1, R);
                const dd SuR = pk_wsum<KERN>(P, ps, 1, r + 1, R);
                const dd SyuR = pk_wsum<KERN>(P, ps, 2, r + 1, R);
                const dd SyL = pk_wsum<KERN>(P, ps, 0, A, r);
                const dd SuL = pk_wsum<KERN>(P, ps, 1, A, r);
                const dd SyuL = pk_wsum<KERN>(P, ps, 2, A, r);
                const int cR = R - r - 1, cL = r - A;
                // sum d  = (SuR - cR delta) + (cL delta - SuL)
                const dd dR = dd_sub(SuR, dd_mul_d_raw(del, (double)cR));
                const dd dL = dd_sub(dd_mul_d_raw(del, (double)cL), SuL);
                s1 = dd_to_d(dd_add(dR, dL));
                // sum y d = (SyuR - delta SyR) + (delta SyL - SyuL)
                const dd yR = dd_sub(SyuR, dd_mul_raw(del, SyR));
                const dd yL = dd_sub(dd_mul_raw(del, SyL), SyuL);
                sy1 = dd_to_d(dd_add(yR, yL));
                sy = dd_to_d(dd_add(SyR, SyL));
            }
            // Eq.(2)-(3) with 0.75 and 1/h^2 cancelled (reading Q5)
            num = fma(hk, sy, -sy1);
            den = fma(hk, (double)c, -s1);
        }
        if (!(den >= 0x1p-20 * hk * (double)c)) {  // reading Q14 ((double)c: exact)
            num = 0.0;
            den = 0.0;
            for (int q = A; q < R; q++) {
                if (q == r) continue;
                const double2 v = xy[q];
                const double d = fabs(v.x - xr);
                const double wt = (KERN == KR_EPANECHNIKOV) ? (h - d) * (h + d) : (h - d);
                num = fma(v.y, wt, num);
                den += wt;
            }
        }
        g = fast_div(num, den);
    }
    const double e = yr - g;
    return e * e;
}

// Boundaries of row r + 1 from row r's at the same bandwidth (sorted x:
// R_{r+1} >= R_r, L_{r+1} >= L_r).  Right: every j in (r+1, R) is inside for
// row r+1; find the first j >= max(R, r+2) outside.  Left: every j <= L is
// outside for row r+1; find the last j <= r outside.  Gallop from the known
// end with steps 1, 2, 4, ... and bisect (typical advance: about one index).
template <int KERN>
__device__ __forceinline__ void window_advance(const double *__restrict__ xs, int n, int r1, double xr1, double h,
                                               int &R, int &L)
{
    int rlo = max(R, r1 + 1) - 1, rhi = 0, rstep = 1;  // rlo: inside for r1 (or r1 itself)
    int llo = L, lhi = 0, lstep = 1;                   // llo: outside for r1
    // Common case first: each boundary moves by 0 or 1 (about one point per
    // row gap).  The four candidates are independent loads -- one memory
    // latency instead of two or three dependent probes per side; xs has
    // +inf sentinels past n, so rlo + 2 <= n + 1 is always readable.
    int rg, lg;
    {
        const double a1 = __ldg(xs + rlo + 1), a2 = __ldg(xs + rlo + 2);
        const int k1 = llo + 1, k2 = llo + 2;  // <= r1 + 1: readable (r1 < n)
        const double b1 = __ldg(xs + k1), b2 = __ldg(xs + k2);
        const int in1 = rlo + 1 <= n && inside<KERN>(a1 - xr1, h);
        const int in2 = rlo + 2 <= n && inside<KERN>(a2 - xr1, h);
        const int out1 = k1 < r1 && !inside<KERN>(xr1 - b1, h);
        const int out2 = k2 < r1 && !inside<KERN>(xr1 - b2, h);
        // right: first outside among rlo+1, rlo+2, else keep galloping from rlo+2
        rhi = !in1 ? rlo + 1 : (!in2 ? rlo + 2 : 0);
        rg = in1 & in2;
        rlo = in1 ? (in2 ? rlo + 2 : rlo + 1) : rlo;
        // left: last outside -- llo+1, llo+2 outside move it; stop at the first inside
        lhi = !out1 ? k1 : (!out2 ? k2 : 0);
        lg = out1 & out2;
        llo = out1 ? (out2 ? k2 : k1) : llo;
        if (rg) rhi = 0;
    }
    while (rg | lg) {
        if (rg) {
            const int k = min(rlo + rstep, n);
            const int in = inside<KERN>(__ldg(xs + k) - xr1, h);
            rlo = in ? k : rlo;
            rhi = in ? rhi : k;
            rstep <<= in;
            rg = in;
        }
        if (lg) {
            const int k = min(llo + lstep, r1);  // r1 itself is "inside" (d = 0)
            const int out = k < r1 && !inside<KERN>(xr1 - __ldg(xs + k), h);
            llo = out ? k : llo;
            lhi = out ? lhi : k;
            lstep <<= out;
            lg = out;
        }
    }
    while (rhi - rlo > 1 || lhi - llo > 1) {
        if (rhi - rlo > 1) {
            const int k = (rlo + rhi) >> 1;
            if (inside<KERN>(__ldg(xs + k) - xr1, h)) rlo = k; else rhi = k;
        }
        if (lhi - llo > 1) {
            const int k = (llo + lhi) >> 1;
            if (!inside<KERN>(xr1 - __ldg(xs + k), h)) llo = k; else lhi = k;
        }
    }
    R = rhi;
    L = llo;
}

// A warp owns 32 * K consecutive sorted rows: lane l the K rows
// base + l K .. base + l K + K - 1, and a chunk of the bandwidth loop.  Per
// bandwidth the lane's first row searches from its previous bandwidth's
// boundaries (window_bounds); each next row starts from its predecessor's
// boundaries at the same bandwidth (window_advance, ~1 probe per side).
template <int KERN, int K>
__global__ void __launch_bounds__(kWinThreads)
window_kernel(const double *__restrict__ xs, const double2 *__restrict__ xy, const double *__restrict__ P,
              int pstride, const double *__restrict__ hg, int m, int n, int row_lo, int row_hi, int ntiles,
              int nbc, const unsigned long long *__restrict__ ymax_bits, double *__restrict__ tileS,
              uint8_t *__restrict__ tileN, int *__restrict__ tile_counter)
{
    pdl_wait();  // krcv_pdl.cuh
    const int lane = threadIdx.x & 31;
    const double o = pfx_origin(xy, n);
    const double ymax = __longlong_as_double((long long)*ymax_bits);
    const int bper = (m + nbc - 1) / nbc;
    const int ps = pstride;
    for (;;) {
        // task = (tile of 32 K rows, chunk of bandwidths): the bandwidth loop is
        // split so that small shards still fill the GPU; a chunk starts its
        // searches cold (from the row itself), later steps from the previous h.
        int task = 0;
        if (lane == 0) task = atomicAdd(tile_counter, 1);
        task = __shfl_sync(0xffffffffu, task, 0);
        if (task >= ntiles * nbc) return;  // warp-uniform
        // chunk-major order: concurrently running warps hold adjacent tiles at
        // the same bandwidths, so their windows (and probes) overlap in L1/L2
        const int chunk = task / ntiles;
        const int tile = task - chunk * ntiles;
        const int b0 = chunk * bper, b1 = min(m, b0 + bper);

        const int i0 = row_lo + tile * 32 * K + lane * K;  // this lane's first row
        WinRow rows[K];
        int nvalid = 0;
#pragma unroll
        for (int k = 0; k < K; k++) {
            const int i = i0 + k;
            nvalid += i < row_hi ? 1 : 0;
            rows[k].r = min(i, row_hi - 1);  // clamped rows do identical work, discarded
            const double2 v = xy[rows[k].r];
            rows[k].xr = v.x;
            rows[k].yr = v.y;
            rows[k].del = two_sum(v.x, -o);  // exact x_r - o
        }
        int kR = 1, kL = 1;  // first row: first offsets not yet known inside
        int gR = cold_step(xs, n, __ldg(hg + b0)), gL = gR;  // first row: gallop steps

        for (int b = b0; b < b1; b++) {
            const double h = __ldg(hg + b);
            const int kR0 = kR, kL0 = kL;
            window_bounds<KERN>(xs, n, rows[0].r, rows[0].xr, h, kR, kL, gR, gL);
            gR = max(1, kR - kR0);
            gL = max(1, kL - kL0);
            int R = rows[0].r + kR, L = rows[0].r - kL;
            double e2 = 0.0;
            int cntM = 0;
#pragma unroll
            for (int k = 0; k < K; k++) {
                if (k > 0) {
                    if (rows[k].r != rows[k - 1].r)
                        window_advance<KERN>(xs, n, rows[k].r, rows[k].xr, h, R, L);
                }
                const int c = R - L - 2;
                if (k < nvalid && c > 0) {  // reading Q6
                    e2 += window_e2<KERN>(rows[k], L + 1, R, c, h, xy, P, ps, ymax);
                    cntM += 1;
                }
            }
            e2 = warp_sum(e2);
            const int cnt = __reduce_add_sync(0xffffffffu, cntM);  // <= 32 K <= 128: fits the u8 slot
            if (lane == 0) {
                tileS[(size_t)b * ntiles + tile] = e2;
                tileN[(size_t)b * ntiles + tile] = (uint8_t)cnt;
            }
        }
    }
}

// Two bandwidths per step: the boundary searches of h_b and h_{b+1} (both
// sides) start from the same previous boundaries and run as four independent
// probe chains in one loop -- twice the memory-level parallelism per warp of
// window_bounds, for a kernel whose time is the latency of dependent probes.
template <int KERN>
__device__ __forceinline__ void window_bounds2(const double *__restrict__ xs, int n, int r, double xr, double ha,
                                               double hb, int kR, int kL, int gR, int gL, int (&kout)[4])
{
    unsigned long long base = reinterpret_cast<unsigned long long>(xs + r);  // see window_bounds
    asm("" : "+l"(base));
    const double *__restrict__ xsr = reinterpret_cast<const double *>(base);
    // chains: 0 right@ha, 1 left@ha, 2 right@hb, 3 left@hb
    int lo[4] = {kR - 1, kL - 1, kR - 1, kL - 1};
    int hi[4] = {0, 0, 0, 0};
    int st[4] = {gR, gL, 2 * gR, 2 * gL};
    int go[4] = {1, 1, 1, 1};
    const int kmax[4] = {n - r, r + 1, n - r, r + 1};
    const double hh[4] = {ha, ha, hb, hb};
    // predicted brackets (see window_bounds): eight independent loads
#pragma unroll
    for (int c = 0; c < 4; c++) {
        const int g = st[c];
        if (g >= 4) {
            const int sg = (int)(3.0f * sqrtf((float)g));
            const int p1 = min(lo[c] + max(1, g - sg), kmax[c]), p2 = min(lo[c] + g + sg, kmax[c]);
            const double d1 = (c & 1) ? xr - __ldg(xsr - p1) : __ldg(xsr + p1) - xr;
            const double d2 = (c & 1) ? xr - __ldg(xsr - p2) : __ldg(xsr + p2) - xr;
            const int in1 = inside<KERN>(d1, hh[c]), in2 = inside<KERN>(d2, hh[c]);
            hi[c] = !in1 ? p1 : (!in2 ? p2 : 0);
            lo[c] = !in1 ? lo[c] : (!in2 ? p1 : p2);
            st[c] = 2 * sg + 1;
            go[c] = in1 & in2;
        }
    }
    while (go[0] | go[1] | go[2] | go[3]) {
#pragma unroll
        for (int c = 0; c < 4; c++) {
            if (go[c]) {
                const int k = min(lo[c] + st[c], kmax[c]);
                const double d = (c & 1) ? xr - __ldg(xsr - k) : __ldg(xsr + k) - xr;
                const int in = inside<KERN>(d, hh[c]);
                lo[c] = in ? k : lo[c];
                hi[c] = in ? hi[c] : k;
                st[c] <<= in;
                go[c] = in;
            }
        }
    }
    while (hi[0] - lo[0] > 1 || hi[1] - lo[1] > 1 || hi[2] - lo[2] > 1 || hi[3] - lo[3] > 1) {
#pragma unroll
        for (int c = 0; c < 4; c++) {
            if (hi[c] - lo[c] > 1) {
                const int k = (lo[c] + hi[c]) >> 1;
                const double d = (c & 1) ? xr - __ldg(xsr - k) : __ldg(xsr + k) - xr;
                if (inside<KERN>(d, hh[c])) lo[c] = k; else hi[c] = k;
            }
        }
    }
#pragma unroll
    for (int c = 0; c < 4; c++) kout[c] = hi[c];
}

template <int KERN>
__global__ void __launch_bounds__(kWinThreads)
window_kernel_b2(const double *__restrict__ xs, const double2 *__restrict__ xy, const double *__restrict__ P,
                 int pstride, const double *__restrict__ hg, int m, int n, int row_lo, int row_hi, int ntiles,
                 int nbc, const unsigned long long *__restrict__ ymax_bits, double *__restrict__ tileS,
                 uint8_t *__restrict__ tileN, int *__restrict__ tile_counter)
{
    pdl_wait();  // krcv_pdl.cuh
    const int lane = threadIdx.x & 31;
    const double o = pfx_origin(xy, n);
    const double ymax = __longlong_as_double((long long)*ymax_bits);
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
        WinRow w;
        w.r = valid ? i : row_hi - 1;  // clamped rows do identical work, discarded
        const double2 v = xy[w.r];
        w.xr = v.x;
        w.yr = v.y;
        w.del = two_sum(v.x, -o);
        int kR = 1, kL = 1, gR = cold_step(xs, n, __ldg(hg + b0)), gL = gR;
        for (int b = b0; b < b1; b += 2) {
            const bool two = b + 1 < b1;
            const double ha = __ldg(hg + b), hb = two ? __ldg(hg + b + 1) : ha;
            int ko[4];
            window_bounds2<KERN>(xs, n, w.r, w.xr, ha, hb, kR, kL, gR, gL, ko);
            gR = max(1, (ko[2] - kR + 1) / 2);
            gL = max(1, (ko[3] - kL + 1) / 2);
            kR = ko[2];
            kL = ko[3];
            double e2a = 0.0, e2b = 0.0;
            bool Ma, Mb;
            {
                const int R = w.r + ko[0], L = w.r - ko[1], c = R - L - 2;
                Ma = valid && c > 0;  // reading Q6
                if (Ma) e2a = window_e2<KERN>(w, L + 1, R, c, ha, xy, P, ps, ymax);
            }
            {
                const int R = w.r + ko[2], L = w.r - ko[3], c = R - L - 2;
                Mb = two && valid && c > 0;
                if (Mb) e2b = window_e2<KERN>(w, L + 1, R, c, hb, xy, P, ps, ymax);
            }
#pragma unroll
            for (int o2 = 16; o2 > 0; o2 >>= 1) {
                e2a += __shfl_xor_sync(0xffffffffu, e2a, o2);
                e2b += __shfl_xor_sync(0xffffffffu, e2b, o2);
            }
            const unsigned balla = __ballot_sync(0xffffffffu, Ma), ballb = __ballot_sync(0xffffffffu, Mb);
            if (lane == 0) {
                tileS[(size_t)b * ntiles + tile] = e2a;
                tileN[(size_t)b * ntiles + tile] = (uint8_t)__popc(balla);
                if (two) {
                    tileS[(size_t)(b + 1) * ntiles + tile] = e2b;
                    tileN[(size_t)(b + 1) * ntiles + tile] = (uint8_t)__popc(ballb);
                }
            }
        }
    }
}

}  // namespace krcv
