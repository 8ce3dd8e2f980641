// krcv_window.cuh -- the window-prefix hot loop with bucket-table boundary
// lookups (a3 + a4 of SURVEY.md §8).
//
// The method (§III P@13614-14984, §IV.B P@21724-22104): for every
// row i and every bandwidth h_b of the ascending grid, the neighbours within
// h_b of x_i, their running sums c, sum y, sum d^2, sum y d^2 (reading Q3),
// the LOO estimate Eq.(2) and the squared error of Eq.(1).  On the globally
// sorted array row r's window at h is the index range [A, R) minus r itself:
//     R = first k > r  with  NOT (xs[k] - x_r < h)   (<= for uniform, Q1)
//     A = first k <= r with       x_r - xs[k] < h
// and the running sums are differences of prefix sums (krcv_prefix.cuh).
//
// What this kernel changes against r01's window_kernel (krcv_prefix.cuh,
// kept for A/B runs as KRCV_WIN=r01): the boundaries are no longer searched
// from the previous bandwidth's (a dependent galloping chain of ~8 probes per
// side), but looked up.  A bucket table over the x range,
//     BT[q] = first k with bkt(xs[k]) >= q,   q = 0 .. Q,
//     bkt(v) = lo32(fma(v, Q / span, 1.5 * 2^52 - x_min Q / span))
// (bkt is round-to-nearest of (v - x_min) Q / span, read from the low mantissa
// word; monotone non-decreasing in v), maps t = x_r + h to a hint
// k0 = BT[bkt(t)]: every k < k0 has xs[k] < t and every k >= BT[bkt(t) + 1]
// has xs[k] > t.  The exact predicate differs from "xs[k] < t" only for
// values within an ulp of t, so four independent probes k0 - 1 .. k0 + 2
// decide the boundary whenever the bucket holds <= 2 points below t; a
// gallop + bisection from the hint covers every other case (ties, crowded
// buckets), so the hint never decides an index, only how fast it is found.
// Q = F n with F = 2^k chosen per call from the data's peak density (the
// smallest x-span of kGapSpan + 1 sorted records, krcv_prefix.cuh), so the
// densest region still averages at most one point per bucket (F <= kBktFmax).
// Sides whose window reaches the end of the data (x_max - x_r < h, resp.
// x_r - x_min < h) take R = n (A = 0) with no lookup at all.
//
// Every (row, bandwidth) is independent, so a warp task is a tile of 32
// consecutive sorted rows (lane = row, coalesced loads) times a chunk of <= 32
// bandwidths, scheduled on persistent warp slots (see win_kernel).
#pragma once

#include <cuda_runtime.h>

#include <climits>
#include <cstdint>

#include "krcv.h"
#include "krcv_pdl.cuh"
#include "krcv_prefix.cuh"

namespace krcv {

#ifndef KRCV_BKT_FMAX
#define KRCV_BKT_FMAX 32
#endif
constexpr int kBktFmax = KRCV_BKT_FMAX;  // buckets per point, at most (build-time A/B)
#ifndef KRCV_BKT_FX
#define KRCV_BKT_FX 1.0                  // (build-time A/B) buckets per point at the peak density
#endif
constexpr int64_t kBktQmax = 1LL << 28;  // buckets, at most
constexpr double kBktMagic = 6755399441055744.0;  // 1.5 * 2^52: fma(.) + magic keeps the integer in the low word
constexpr int kBktFillThreads = 256;

// Table parameters, written by bkt_fill_kernel's first thread, read by the
// window kernel (both compute them from the same inputs).
struct BktParams {
    double invw;  // Q / span
    double C;     // kBktMagic - x_min Q / span
    int Q;        // buckets 0 .. Q
    int F;
};

__device__ __forceinline__ int bkt_raw(double v, double invw, double C)
{
    return __double2loint(fma(v, invw, C));
}

// Parameters of the table for this call: F from the peak density.
__device__ __forceinline__ BktParams bkt_params_of(double lo, double hi, int n, unsigned long long gb)
{
    BktParams p;
    const double span = hi - lo;
    int F = 1;
    if (gb != 0ull && span > 0.0) {
        const double gap = __longlong_as_double((long long)~gb);  // min x-span of kGapSpan + 1 records
        // ratio of the peak density kGapSpan / gap to the mean (n - 1) / span:
        // F = the next power of two, at most one point per bucket where the data
        // is densest (uniform x: F = 2; a larger table costs L2 capacity, which
        // the C4 working set needs -- profiles/r02f_*)
        const double ratio = gap > 0.0 ? KRCV_BKT_FX * (double)kGapSpan * span / (gap * (double)(n - 1)) : 1e300;
        while (F < kBktFmax && (double)F < ratio) F <<= 1;
    }
    int64_t Q = (int64_t)F * n;
    if (Q > kBktQmax) Q = kBktQmax;
    p.F = F;
    p.Q = (int)Q;
    p.invw = span > 0.0 ? (double)Q / span : 0.0;
    p.C = kBktMagic - lo * p.invw;
    return p;
}

__device__ __forceinline__ BktParams bkt_params(const double *__restrict__ xs, int n,
                                                const unsigned long long *__restrict__ gap_bits)
{
    return bkt_params_of(xs[0], xs[n - 1], n, *gap_bits);
}

// Fused O(n) build for a problem whose 256-record prefix tiles all fit on
// the GPU at once (ntiles <= #SMs, so every CTA is co-resident), one record
// per thread.  It is latency-bound (two warps per SM sub-partition, long
// dependent dd chains), so every step is done once:
//   1. the record's moment terms (kept in registers), the warp's inclusive dd
//      scan of them, the density statistic and max|y|; the warp totals give
//      the tile's warp offsets and total in one fixed-order pass (5 threads,
//      one per moment), the total -> tot[k][tile];
//   2. a grid barrier (arrival counter, zeroed by the call's status memset);
//   3. the tile's offset: the totals of the earlier tiles in fixed order
//      (strided per thread, butterfly per warp, warp partials in order);
//      P[j] = offset + warp offset + the lane's exclusive scan; records, xs;
//   4. this tile's stretch of the bucket table: q in (bkt(x_{j0-1}),
//      bkt(x_{j1-1})] (from 0 for the first tile, to Q for the last), BT[q] =
//      the first of the tile's records with bucket >= q, by a binary search
//      over the tile's bucket ids in shared memory -- the table
//      bkt_fill_kernel builds.
// One launch instead of three; every sum in a fixed order (bit-reproducible;
// its rounding differs from the two-phase build's in the last dd bits, as the
// two-phase build's differs from the one-CTA build's).
constexpr int kFusedPfxThreads = kPfxThreads;  // one record per thread (ITEMS = 1)

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned *p)
{
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

template <int KERN>
__global__ void __launch_bounds__(kFusedPfxThreads)
pfx_fused_kernel(const double2 *__restrict__ xy, int n, double2 *__restrict__ tot, int ntiles,
                 unsigned long long *__restrict__ ymax_bits, unsigned long long *__restrict__ gap_bits,
                 double *__restrict__ P, int pstride, double *__restrict__ xs, int *__restrict__ BT,
                 BktParams *__restrict__ prm, unsigned *__restrict__ arrive)
{
    pdl_wait();  // krcv_pdl.cuh
    constexpr int K = NMom<KERN>::v;
    constexpr int W = kFusedPfxThreads / 32;
    __shared__ double2 wtot[K][W];  // warp totals, then the warps' exclusive offsets
    __shared__ double2 base_s[K];
    __shared__ int sA[kFusedPfxThreads];
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    const int tile = blockIdx.x;
    const int j = tile * kFusedPfxThreads + t;
    if (tile == 0 && t < kPad) {
        xs[-1 - t] = -INFINITY;
        xs[n + t] = INFINITY;
    }
    // 1. terms, warp scan, statistics
    const double o = pfx_origin(xy, n);
    dd tm[kPfxMoments], inc[kPfxMoments];
    double xj = 0.0, ym = 0.0, gmin = INFINITY;
    if (j < n) {
        const double2 v = xy[j];
        xj = v.x;
        ym = fabs(v.y);
        gap_stat(xy, n, j, gmin);
        moment_terms<KERN>(v.x, v.y, o, tm);
    } else {
#pragma unroll
        for (int k = 0; k < K; k++) tm[k] = dd{0.0, 0.0};
    }
#pragma unroll
    for (int k = 0; k < K; k++) inc[k] = tm[k];
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            const dd u = shfl_up_dd(inc[k], d);
            if (lane >= d) inc[k] = dd_add(u, inc[k]);
        }
    }
    if (lane == 31) {
#pragma unroll
        for (int k = 0; k < K; k++) st_dd(&wtot[k][w], inc[k]);
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) ym = fmax(ym, __shfl_xor_sync(0xffffffffu, ym, d));
    if (lane == 0 && ym > 0.0) atomicMax(ymax_bits, (unsigned long long)__double_as_longlong(ym));
    gap_publish(gmin, gap_bits);
    __syncthreads();
    if (t < K) {  // warp offsets (exclusive, in warp order) and the tile total
        dd run = dd{0.0, 0.0};
        for (int q = 0; q < W; q++) {
            const dd v = ld_dd(&wtot[t][q]);
            st_dd(&wtot[t][q], run);
            run = q == 0 ? v : dd_add(run, v);
        }
        st_dd(tot + (size_t)t * ntiles + tile, run);
    }
    __syncthreads();
    // 2. grid barrier
    if (t == 0) {
        __threadfence();
        atomicAdd(arrive, 1u);
        while (ld_acquire_u32(arrive) < gridDim.x) __nanosleep(32);
        __threadfence();
    }
    __syncthreads();
    // 3. the tile's offset, the records
    {
        dd a[kPfxMoments];
#pragma unroll
        for (int k = 0; k < K; k++) {
            a[k] = dd{0.0, 0.0};
            for (int q = t; q < tile; q += kFusedPfxThreads) {
                const double2 *pq = tot + (size_t)k * ntiles + q;
                a[k] = dd_add(a[k], dd{__ldcg(&pq->x), __ldcg(&pq->y)});
            }
        }
        if (tile > 32 * w) {  // warps whose strided range holds earlier tiles
#pragma unroll
            for (int d = 16; d > 0; d >>= 1) {
#pragma unroll
                for (int k = 0; k < K; k++) a[k] = dd_add(a[k], shfl_xor_dd(a[k], d));
            }
        }
        __shared__ double2 psum[K][W];
        if (lane == 0) {
#pragma unroll
            for (int k = 0; k < K; k++) st_dd(&psum[k][w], a[k]);
        }
        __syncthreads();
        if (t < K) {
            dd b = dd{0.0, 0.0};
            const int nw = min(W, (tile + 31) / 32);
            for (int q = 0; q < nw; q++) b = dd_add(b, ld_dd(&psum[t][q]));
            st_dd(&base_s[t], b);
        }
        __syncthreads();
    }
#pragma unroll
    for (int k = 0; k < K; k++) {
        const dd u = shfl_up_dd(inc[k], 1);
        const dd ex = lane == 0 ? dd{0.0, 0.0} : u;
        if (j <= n) pk_store<KERN>(P, pstride, k, j, dd_add(dd_add(ld_dd(&base_s[k]), ld_dd(&wtot[k][w])), ex));
    }
    if (j <= n) pk_store_index<KERN>(P, pstride, j);
    if (j < n) xs[j] = xj;
    // 4. bucket table
    if (!BT) return;
    const BktParams p = bkt_params_of(__ldg(&xy[0].x), __ldg(&xy[n - 1].x), n, __ldcg(gap_bits));
    if (tile == 0 && t == 0) *prm = p;
    auto A = [&](double v) { return min(max(bkt_raw(v, p.invw, p.C), 0), p.Q); };
    const int j0 = tile * kFusedPfxThreads, j1 = min(j0 + kFusedPfxThreads, n), cnt = j1 - j0;
    sA[t] = t < cnt ? A(xj) : INT_MAX;
    __syncthreads();
    const int qlo = j0 == 0 ? 0 : A(__ldg(&xy[j0 - 1].x)) + 1;
    const int qhi = j1 == n ? p.Q : sA[cnt - 1];
    for (int q = qlo + t; q <= qhi; q += kFusedPfxThreads) {
        int lo = 0, hi = cnt;
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (sA[mid] >= q) hi = mid; else lo = mid + 1;
        }
        BT[q] = j0 + lo;
    }
}

// BT[q] = #{k : bkt(xs[k]) < q} for q = 0 .. Q: the merge of the sorted
// bucket ids A[k] = clamp(bkt(xs[k]), 0, Q) with the sequence 0 .. Q (A[k]
// goes first iff A[k] < q), cut by merge path at two levels so long runs of
// empty buckets (the sparse tail of a heavy-tailed x) are spread evenly:
// a CTA takes kBktTile consecutive merged items, its two warps find the
// tile's ends on the diagonals (32 probes per round: log32 rounds of
// dependent loads instead of log2), the CTA stages the tile's bucket ids in
// shared memory, and each thread merges kBktItems items from its own split
// (a binary search in shared memory).  Grid-stride over tiles.
constexpr int kBktItems = 16;
constexpr int kBktTile = kBktFillThreads * kBktItems;

// smallest i in [lo, hi] with p(i) true (p monotone, p(hi) taken as true),
// found by all 32 lanes of a warp together; every lane returns it
template <class Pred>
__device__ __forceinline__ int64_t warp_first_true(Pred p, int64_t lo, int64_t hi, int lane)
{
    while (hi > lo) {
        // lane l tests the end of sub-range l of ceil(len / 32) items; lane
        // 31's sub-range ends at hi (true by definition)
        const int64_t step = (hi - lo + 31) / 32;
        const int64_t q = lo + (int64_t)(lane + 1) * step - 1;
        const bool t = lane == 31 || q >= hi || p(q);
        const int f = __ffs(__ballot_sync(0xffffffffu, t)) - 1;
        const int64_t end = lo + (int64_t)(f + 1) * step - 1;
        hi = (f == 31 || end > hi) ? hi : end;
        lo = lo + (int64_t)f * step;
    }
    return hi;
}

__global__ void __launch_bounds__(kBktFillThreads)
bkt_fill_kernel(const double *__restrict__ xs, int n, const unsigned long long *__restrict__ gap_bits,
                int *__restrict__ BT, BktParams *__restrict__ prm)
{
    pdl_wait();  // krcv_pdl.cuh
    __shared__ int sA[kBktTile];
    __shared__ int sBT[kBktTile];  // the tile's table entries, stored coalesced at the end
    __shared__ int64_t split[2];
    const BktParams p = bkt_params(xs, n, gap_bits);
    if (blockIdx.x == 0 && threadIdx.x == 0) *prm = p;
    const int Q = p.Q;
    auto A = [&](int64_t k) { return (int64_t)min(max(bkt_raw(xs[k], p.invw, p.C), 0), Q); };
    const int64_t total = (int64_t)n + Q + 1;
    const int t = threadIdx.x, lane = t & 31, w = t >> 5;
    for (int64_t D0 = (int64_t)blockIdx.x * kBktTile; D0 < total; D0 += (int64_t)gridDim.x * kBktTile) {
        const int64_t D1 = D0 + kBktTile < total ? D0 + kBktTile : total;
        if (w < 2) {
            // split of the first d merged items: i from A, d - i from 0..Q;
            // the smallest i with A[i] >= d - i - 1 (monotone in i)
            const int64_t d = w == 0 ? D0 : D1;
            const int64_t lo = d - (Q + 1) > 0 ? d - (Q + 1) : 0;
            const int64_t hi = d < n ? d : n;
            const int64_t s = warp_first_true([&](int64_t i) { return A(i) >= d - i - 1; }, lo, hi, lane);
            if (lane == 0) split[w] = s;
        }
        __syncthreads();
        const int64_t i0 = split[0], i1 = split[1];
        const int cnt = (int)(i1 - i0);  // <= kBktTile
        for (int k = t; k < cnt; k += kBktFillThreads) sA[k] = (int)A(i0 + k);
        __syncthreads();
        // this thread's items: local diagonal dl = t kBktItems of the tile
        const int dl = t * kBktItems;
        const int64_t d = D0 + dl;
        const int jn = (int)(D1 - D0) - cnt;  // bucket items of the tile: q = D0 - i0 ..
        const int64_t jb = D0 - i0;
        if (d < D1) {
            int lo = dl - jn > 0 ? dl - jn : 0, hi = dl < cnt ? dl : cnt;
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if ((int64_t)sA[mid] >= d - (i0 + mid) - 1) hi = mid; else lo = mid + 1;
            }
            int i = lo;
            int64_t j = d - (i0 + i);
            for (int s = 0; s < kBktItems && D0 + dl + s < D1; s++) {
                if (i < cnt && (int64_t)sA[i] < j) {
                    i++;
                } else {
                    sBT[j - jb] = (int)(i0 + i);
                    j++;
                }
            }
        }
        __syncthreads();
        for (int k = t; k < jn; k += kBktFillThreads) BT[jb + k] = sBT[k];
        __syncthreads();  // sA / sBT / split reused by the next tile
    }
}

// ---------------------------------------------------------------------------
// Anchored records (Epanechnikov fast path; DESIGN.md §6.2 "anchored
// records").  The fast path reads hi words of prefix differences and shifts
// them to the row: its error is eps times the magnitudes it combines -- the
// prefix values at A and R, accumulated from index 0 about the global origin
// o, and (x_r - o)^2 per window point -- so rows far from o at small h fail
// the bound and take the dd path (18 % of (row, b) at C2-C4, 36 % at C5).  J
// anchors s_j = floor((2 j + 1) n / (2 J)) (the centres of J equal index
// regions) each get a copy of the hi words anchored there and taken about
// o_j = xs[s_j]:
//     V_j[k] = sum_{l in [s_j, k)} term_j(l)     (k >= s_j; minus the sum
//              over [k, s_j) below), term_j = (y, u', u'^2, y u', y u'^2),
//     u' = x - o_j,
// computed from the global dd records P[k] - P[s_j] (S) by the exact shift
// Delta = o_j - o (dd), c = k - s_j:
//     V_y = S_y, V_u = S_u - c Delta, V_uu = S_uu - 2 Delta S_u + c Delta^2,
//     V_yu = S_yu - Delta S_y, V_yuu = S_yuu - 2 Delta S_yu + Delta^2 S_y,
// normalised and rounded to nearest.  A task's rows use the copy of their
// region: their prefix magnitudes and shift are local.  Error of a stored
// word beyond its rounding: the dd arithmetic's and the difference of the
// two dd prefix values' own scan errors, bounded by
// kappa(k) Gamma = (|k - s_j| + 2048) 2^-100 times the operand magnitudes
// Gamma of the value (the fixed-order tiled scan accumulates its error
// between s_j and k); where kappa Gamma > 2^-57 |V| in any of the five planes
// the copy holds NaN at k (the fast test fails, the window is recomputed
// from the global dd records), so every stored word is within
// (eps/2 + 2^-57) |V| of the exact anchored sum -- inside the fast-path
// bound's slack (kFastSlack = 16 eps).  The dd path is unchanged.
// Copy j occupies virtual indices j S .. j S + n of one blocked record array
// (S = pk_slots), so the fast path only adds j S to its two indices.
constexpr int kAncMax = 16;            // anchors, at most (o_j table: status bytes 96-223)
constexpr int64_t kAncMaxN = 1LL << 25;  // no anchors above (their copies: 40 kAncMax B per point)
constexpr int64_t kAncMinN = 50000;    // no anchors below (measured: no gain at C2, profiles/r02/r02aq_*)
constexpr double kAncHotBytes = 96.0 * 1024 * 1024;  // anchored copies hot in L2 under one band, at most
constexpr int kAncThreads = 256;
__host__ __device__ __forceinline__ int anc_s(int j, int J, int n)
{
    return (int)(((int64_t)(2 * j + 1) * n) / (2 * J));
}
__host__ __device__ __forceinline__ int anc_of(int r, int J, int n)
{
    const int j = (int)(((int64_t)r * J) / n);
    return j < J ? j : J - 1;
}

// One thread per (index k, anchor j) for the nj anchors j0 .. j0 + nj - 1:
// block b covers indices (b / nj) 256 .. + 255 of copy j = j0 + b mod nj, so
// the copies of a stretch of records are written together and P[k] is read
// from DRAM once (anchor-major blocks re-streamed P J times: C4 J = 8 build
// 94 -> 274 us).  OJ[j] = o_j (the window kernel's table).
template <int KERN>
__global__ void __launch_bounds__(kAncThreads)
anchor_kernel(const double *__restrict__ xs, const double *__restrict__ P, int ps, int n, int J, int j0, int nj,
              double *__restrict__ PA, double *__restrict__ OJ)
{
    static_assert(PfxRec<KERN>::S == 5 && !kRecAos, "anchored records: the Epanechnikov blocked layout");
    pdl_wait();  // krcv_pdl.cuh
    const int j = j0 + (int)(blockIdx.x % (unsigned)nj);
    const int s = anc_s(j, J, n);
    const double o = xs[n >> 1];      // pfx_origin: the median sorted record
    const dd D = two_sum(xs[s], -o);  // o_j - o, exact
    const dd D2 = dd_mul(D, D);
    const double aD = fabs(D.hi) * (1.0 + 0x1p-52), aD2 = aD * aD * (1.0 + 0x1p-51);  // >= |Delta|, Delta^2
    if (blockIdx.x < (unsigned)nj && threadIdx.x == 0) OJ[j] = xs[s];
    const int k = (int)(blockIdx.x / (unsigned)nj) * blockDim.x + threadIdx.x;
    if (k > n) return;
    dd S[5];
    double M[5];
#pragma unroll
    for (int q = 0; q < 5; q++) {
        const dd a = pk_dd<KERN>(P, ps, q, k), b = pk_dd<KERN>(P, ps, q, s);
        S[q] = dd_sub(a, b);
        M[q] = fabs(a.hi) + fabs(a.lo) + fabs(b.hi) + fabs(b.lo);
    }
    const double c = (double)(k - s);  // exact
    const double ac = fabs(c);
    double V[5];
    V[0] = S[0].hi;
    V[1] = dd_sub(S[1], dd_mul_d(D, c)).hi;
    V[2] = dd_add(dd_sub(S[2], dd_twice(dd_mul(D, S[1]))), dd_mul_d(D2, c)).hi;
    V[3] = dd_sub(S[3], dd_mul(D, S[0])).hi;
    V[4] = dd_add(dd_sub(S[4], dd_twice(dd_mul(D, S[3]))), dd_mul(D2, S[0])).hi;
    // operand magnitudes Gamma of each value (upper bounds), kappa(k) Gamma <= 2^-57 |V| or NaN
    const double G[5] = {M[0], M[1] + ac * aD, M[2] + 2.0 * aD * M[1] + ac * aD2, M[3] + aD * M[0],
                         M[4] + 2.0 * aD * M[3] + aD2 * M[0]};
    const double kap = (ac + 2048.0) * 0x1p-100 * (1.0 + 0x1p-48);
    bool ok = true;
#pragma unroll
    for (int q = 0; q < 5; q++) ok = ok && kap * G[q] * (1.0 + 0x1p-50) <= 0x1p-57 * fabs(V[q]);
    const int v = j * (int)pk_slots(ps) + k;  // virtual index of (copy j, k)
#pragma unroll
    for (int q = 0; q < 5; q++) PA[pk_off<KERN>(q, v)] = ok ? V[q] : __longlong_as_double(0x7ff8000000000000LL);
}

// First k in [lo, hi] with p(k) true, p monotone (false ... true), p(hi)
// true, and p(lo - 1) false wherever it is read (the +-inf sentinels and row
// r make that hold for both sides).  Four probes around the hint k0 settle
// the common case; otherwise gallop from the hint in the direction the probes
// point, then bisect.  Exact for any hint.
template <class Pred>
__device__ __forceinline__ int first_true(Pred p, int lo, int hi, int k0)
{
    const int k = min(max(k0, lo), hi);
    const bool pa = p(k - 1), pb = p(k), pc = p(k + 1), pd = p(k + 2);
    if (!pa && pd) return k + (pb ? 0 : (pc ? 1 : 2));
    int a, b;  // p(a) false (a >= lo - 1), p(b) true
    if (pa) {  // boundary at or below k - 1: gallop down
        b = k - 1;
        int step = 1;
        a = b - 1;
        while (a >= lo && p(a)) {
            b = a;
            step <<= 1;
            a = b - step;
        }
        a = max(a, lo - 1);
    } else {   // p(k + 2) false: gallop up
        a = k + 2;
        int step = 1;
        b = min(a + 1, hi);
        while (b < hi && !p(b)) {
            a = b;
            step <<= 1;
            b = min(a + step, hi);
        }
    }
    while (b - a > 1) {
        const int mid = (a + b) >> 1;
        if (p(mid)) b = mid; else a = mid;
    }
    return b;
}

constexpr int kWin2Warps = 4;
constexpr int kWin2Threads = kWin2Warps * 32;
#ifndef KRCV_WIN2_ROWS
#define KRCV_WIN2_ROWS 2
#endif
constexpr int kWin2Rows = KRCV_WIN2_ROWS;  // tiles of 32 rows per task = rows per lane (1 or 2)
#ifndef KRCV_WIN2_ACC
#define KRCV_WIN2_ACC 1
#endif
constexpr int kWin2Acc = KRCV_WIN2_ACC;  // running sums per lane (build-time A/B: 1 or 2)
constexpr int kWin2Chunk = 32 * kWin2Acc;  // bandwidths per task, at most (lane (b - b0) % 32 keeps b's sum)
// CTAs per SM the register allocation must allow: 8 -> 64 registers, 32
// warps per SM (measured faster than 6 -> 80 and 4 -> 128 registers: the
// kernel is latency-bound, profiles/r02d_*, r02e_*).  KRCV_WIN2_MINB at build
// time overrides (tuning runs).
#ifndef KRCV_WIN2_MINB
#define KRCV_WIN2_MINB 8
#endif
constexpr int kWin2MinBlocks = KRCV_WIN2_MINB;

// Schedule.  Task k = (chunk c = k / npairs of <= 32 bandwidths, tile pair
// t = k % npairs: 64 consecutive sorted rows, two per lane), chunk-major.  The grid is
// persistent: S = gridDim.x * kWin2Warps warp slots, slot s runs tasks s, s + S,
// s + 2S, ... (static, no atomics).  So the tasks in flight at any moment are S
// consecutive tiles of one chunk -- a band of 32 S rows whose windows at
// nearby bandwidths touch a band of the sorted arrays that stays in L2 (an
// earlier schedule with every row block in flight touched the whole array per
// bandwidth and read 7-12 GB from DRAM per C4 launch, profiles/r02f_*,
// r02g_*).  Per (tile, bandwidth) the squared errors are summed by a fixed
// butterfly and lane b - b0 adds the sum to the slot's running sum for b over
// the slot's consecutive tasks of the same chunk; the sum is written once per
// (slot, chunk) to tileS[b][s] (tileN likewise).  reduce_slots_kernel adds the
// slots of each bandwidth in slot order: bit-reproducible, and S m partials
// instead of one per (tile, bandwidth) (the per-tile partials
// were 6x the algorithmic DRAM bytes at C4).
// No shared memory: the probes and prefix records live in L1, and shared
// memory a CTA reserves is taken from the L1 carve-out (a shared-memory batch
// reduction measured 12% slower at C4 for that reason, profiles/r02e_*).
// Squared LOO error of one row at bandwidth h (0 if the row is invalid or has
// an empty window, reading Q6), M through *M.
template <int KERN>
__device__ __forceinline__ double row_e2(const WinRow &w, bool valid, double dmax, double dmin, double h,
                                         const double *__restrict__ xs, const double2 *__restrict__ xy,
                                         const double *__restrict__ P, int pstride, const int *__restrict__ BT,
                                         double invw, double C, int Q, int n, double ymax, bool &M,
                                         const WinAnc *an = nullptr)
{
    const int r = w.r;
    const double xr = w.xr;
    int R = n, A = 0;
    if (!inside<KERN>(dmax, h)) {  // window ends inside the data: look R up
        const int k0 = __ldg(BT + min(max(bkt_raw(xr + h, invw, C), 0), Q));
        R = first_true([&](int q) { return !inside<KERN>(__ldg(xs + q) - xr, h); }, r + 1, n, k0);
    }
    if (!inside<KERN>(dmin, h)) {
        const int k0 = __ldg(BT + min(max(bkt_raw(xr - h, invw, C), 0), Q));
        A = first_true([&](int q) { return inside<KERN>(xr - __ldg(xs + q), h); }, 0, r, k0);
    }
    const int c = R - A - 1;
    M = valid && c > 0;  // reading Q6
    return M ? window_e2<KERN>(w, A, R, c, h, xy, P, pstride, ymax, an) : 0.0;
}

// Task-schedule constants of a win_kernel launch (host-computed): npairs
// tile pairs per chunk, ntasks = npairs nbc, S / npairs and S mod npairs for
// the incremental task index (S = the grid's warp slots).
struct Win2Sched {
    int npairs, s_div, s_mod;
    long long ntasks;
};

template <int KERN, bool ANC>
__global__ void __launch_bounds__(kWin2Threads, kWin2MinBlocks)
win_kernel(const double *__restrict__ xs, const double2 *__restrict__ xy, const double *__restrict__ P, int pstride,
           const int *__restrict__ BT, const BktParams *__restrict__ prm, const double *__restrict__ hg, int m,
           int n, int row_lo, int row_hi, int ntiles, int BC, int nbc,
           const unsigned long long *__restrict__ ymax_bits, double *__restrict__ tileS,
           uint32_t *__restrict__ tileN, const double *__restrict__ PA, int J, int j0, int j1,
           const double *__restrict__ OJ, Win2Sched sc)
{
    static_assert(!ANC || KERN == KR_EPANECHNIKOV, "anchored records: Epanechnikov only");
    pdl_wait();  // krcv_pdl.cuh
    const int lane = threadIdx.x & 31;
    const int S = gridDim.x * kWin2Warps;
    const int slot = blockIdx.x * kWin2Warps + (threadIdx.x >> 5);
    const double o = pfx_origin(xy, n);
    const double ymax = __longlong_as_double((long long)*ymax_bits);
    const double xmin = xs[0], xmax = xs[n - 1];
    const double invw = prm->invw, C = prm->C;
    const int Q = prm->Q;
    // anchored records (ANC): the anchor of a task is the region of its middle row (any anchor is exact)
    const double rJ = (double)J / (double)n;
    const int Sv = ANC ? (int)pk_slots(pstride) : 0;  // virtual indices per anchored copy
    // a task is kWin2Rows adjacent tiles (2: 64 rows, two rows per lane
    // sharing one butterfly per bandwidth)
    // schedule constants from the host (kernel parameters: the 64-register
    // kernel would otherwise recompute S mod npairs per task)
    const int npairs = sc.npairs;
    const int64_t ntasks = sc.ntasks;
    int cur = -1;  // chunk of the running sums
    double acc[kWin2Acc];
    uint32_t cnt[kWin2Acc];
#pragma unroll
    for (int a = 0; a < kWin2Acc; a++) {
        acc[a] = 0.0;
        cnt[a] = 0;
    }
    // task k = slot + i S -> (chunk, t) advanced incrementally (no 64-bit
    // division per task)
    int kchunk = slot / npairs, kt = slot - kchunk * npairs;
    for (int64_t k = slot;; k += S) {
        const int chunk = k < ntasks ? kchunk : nbc;  // warp-uniform
        if (chunk != cur) {  // flush the previous chunk's sums, start the next
#pragma unroll
            for (int a = 0; a < kWin2Acc; a++) {
                const int bw = cur * BC + 32 * a + lane;
                if (cur >= 0 && bw < min(m, (cur + 1) * BC)) {
                    tileS[(size_t)bw * S + slot] = acc[a];
                    tileN[(size_t)bw * S + slot] = cnt[a];
                }
                acc[a] = 0.0;
                cnt[a] = 0;
            }
            if (chunk >= nbc) return;
            cur = chunk;
        }
        const int t = kt;
        kt += sc.s_mod;
        kchunk += sc.s_div;
        if (kt >= npairs) {
            kt -= npairs;
            kchunk += 1;
        }
        const int b0 = chunk * BC, b1 = min(m, b0 + BC);
        WinRow w0, w1;
        int joff = 0;
        double dla0 = 0.0, dla1 = 0.0;
        bool v0, v1 = false;
        double dmax0, dmin0, dmax1 = 0.0, dmin1 = 0.0;
        {
            const int i = row_lo + t * 32 * kWin2Rows + lane;
            v0 = i < row_hi;
            w0.r = v0 ? i : row_hi - 1;  // clamped rows do identical work, discarded
            const double2 v = xy[w0.r];
            w0.xr = v.x;
            w0.yr = v.y;
            w0.del = ANC ? dd{0.0, 0.0} : two_sum(v.x, -o);  // exact x_r - o (the anchored dd path recomputes it)
            dmax0 = xmax - v.x;
            dmin0 = v.x - xmin;
        }
        if (kWin2Rows == 2) {
            const int i = row_lo + t * 64 + 32 + lane;
            v1 = i < row_hi;
            w1.r = v1 ? i : row_hi - 1;
            const double2 v = xy[w1.r];
            w1.xr = v.x;
            w1.yr = v.y;
            w1.del = ANC ? dd{0.0, 0.0} : two_sum(v.x, -o);
            dmax1 = xmax - v.x;
            dmin1 = v.x - xmin;
        }
        if (ANC) {  // warp-uniform: the task's anchor, among the copies built for rows [row_lo, row_hi)
            const int mid = min(row_lo + t * 32 * kWin2Rows + 16 * kWin2Rows, row_hi - 1);
            const int j = min(j1, max(j0, (int)((double)mid * rJ)));
            const double oj = __ldg(OJ + j);
            joff = j * Sv;
            dla0 = w0.xr - oj;
            dla1 = w1.xr - oj;
        }
        for (int b = b0; b < b1; b++) {
            const double h = __ldg(hg + b);
            bool M0, M1;
            const WinAnc an0{PA, joff, dla0, o}, an1{PA, joff, dla1, o};
            double e2 = row_e2<KERN>(w0, v0, dmax0, dmin0, h, xs, xy, P, pstride, BT, invw, C, Q, n, ymax, M0,
                                     ANC ? &an0 : nullptr);
            M1 = false;
            if (kWin2Rows == 2)
                e2 += row_e2<KERN>(w1, v1, dmax1, dmin1, h, xs, xy, P, pstride, BT, invw, C, Q, n, ymax, M1,
                                   ANC ? &an1 : nullptr);
            e2 = warp_sum(e2);  // fixed butterfly: every lane holds the task's sum
            const uint32_t nb = __popc(__ballot_sync(0xffffffffu, M0)) +
                                (kWin2Rows == 2 ? __popc(__ballot_sync(0xffffffffu, M1)) : 0u);
            const int bl = b - b0;
            if (kWin2Acc == 1) {  // bl < 32: lane bl keeps bandwidth b's sums
                if (lane == bl) {
                    acc[0] += e2;
                    cnt[0] += nb;
                }
            } else if (lane == (bl & 31)) {
#pragma unroll
                for (int a = 0; a < kWin2Acc; a++)
                    if ((bl >> 5) == a) {
                        acc[a] += e2;
                        cnt[a] += nb;
                    }
            }
        }
    }
}

}  // namespace krcv
