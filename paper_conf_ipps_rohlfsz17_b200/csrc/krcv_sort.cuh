// krcv_sort.cuh -- ordering step for shards up to
// kRankSortMaxN rows, fused with a1 (pack + validation) and the gather.
//
// The paper orders each row's distances with a per-thread QuickSort
// (P@20542); here ONE global order of (x, original index) serves every row
// (DESIGN.md §7).  For small n the CUB onesweep radix sort is latency-bound
// (~10 us per 8-bit pass, 8 passes for 64-bit keys; profiles/), so:
//
//   K1 chunk_sort_kernel:  each CTA packs kChunk records (order-preserving
//      u64 key of x, u32 index), counts non-finite inputs and bad grid
//      entries, and sorts the chunk in registers/shared memory
//      (cub::BlockMergeSort::StableSort, so ties stay in index order);
//   K2 rank_count_kernel: one CTA per ordered chunk pair (c, cc): the count
//      of chunk cc's records that compare less than each record of chunk c
//      (fixed-depth binary searches), added to the record's rank;
//   K3 rank_scatter_kernel: writes (x, y) straight to that rank in the
//      sorted array -- no merge passes, no separate gather.  (key, index)
//      pairs are unique, so the order is total and identical to a stable
//      sort by x.
#pragma once

#include "krcv_pdl.cuh"

#include <cuda_runtime.h>

#include <cstdint>

#include <cub/block/block_merge_sort.cuh>


#include "krcv_sweep.cuh"

namespace krcv {

// Chunk configurations (threads x items): 256x4 = 1024, 256x8 = 2048,
// 512x8 = 4096 records per CTA (chunk_config()).  kChunk is the largest, used
// to pad the workspace arrays so every configuration fits.
constexpr int kChunk = 4096;
constexpr int64_t kRankSortMaxN = 131072;

__device__ __forceinline__ uint64_t order_key(double v)
{
    // IEEE-754 total order on non-NaN values as an unsigned integer.
    uint64_t u = static_cast<uint64_t>(__double_as_longlong(v));
    return (u & 0x8000000000000000ull) ? ~u : (u | 0x8000000000000000ull);
}

__device__ __forceinline__ bool kv_less(uint64_t ka, uint32_t ia, uint64_t kb, uint32_t ib)
{
    return ka < kb || (ka == kb && ia < ib);
}

struct KeyLess {
    __device__ __forceinline__ bool operator()(const uint64_t &a, const uint64_t &b) const { return a < b; }
};

template <int kChunkThreads, int kChunkItems>
__global__ void __launch_bounds__(kChunkThreads)
chunk_sort_kernel(const double *__restrict__ x, const double *__restrict__ y, int n,
                  const double *__restrict__ h, int m, uint64_t *__restrict__ keys,
                  uint32_t *__restrict__ khi, uint32_t *__restrict__ idx, int *__restrict__ rank,
                  unsigned *__restrict__ status)
{
    constexpr int kChunk = kChunkThreads * kChunkItems;
    using BMS = cub::BlockMergeSort<uint64_t, kChunkThreads, kChunkItems, uint32_t>;
    __shared__ typename BMS::TempStorage ts;
    const int base = blockIdx.x * kChunk;
    uint64_t k[kChunkItems];
    uint32_t v[kChunkItems];
    unsigned bad = 0;
#pragma unroll
    for (int q = 0; q < kChunkItems; q++) {  // blocked arrangement: index order per thread
        const int g = base + threadIdx.x * kChunkItems + q;
        if (g < n) {
            const double xv = x[g], yv = y[g];
            bad += (!isfinite(xv) || !isfinite(yv)) ? 1u : 0u;
            k[q] = order_key(xv);
            v[q] = (uint32_t)g;
        } else {
            k[q] = ~0ull;  // padding sorts last
            v[q] = 0xffffffffu;
        }
    }
    unsigned gbad = 0;
    if (blockIdx.x == 0)
        for (int b = threadIdx.x; b < m; b += kChunkThreads) {
            const double hb = h[b];
            gbad += (!isfinite(hb) || !(hb > 0.0) || (b > 0 && hb < h[b - 1])) ? 1u : 0u;
        }
    if (bad) atomicAdd(&status[1], bad);
    if (gbad) atomicAdd(&status[0], gbad);
    BMS(ts).StableSort(k, v, KeyLess());  // stable: equal keys keep index order
#pragma unroll
    for (int q = 0; q < kChunkItems; q++) {
        keys[base + threadIdx.x * kChunkItems + q] = k[q];
        khi[base + threadIdx.x * kChunkItems + q] = (uint32_t)(k[q] >> 32);
        rank[base + threadIdx.x * kChunkItems + q] = threadIdx.x * kChunkItems + q;  // + counts (K2)
        idx[base + threadIdx.x * kChunkItems + q] = v[q];
    }
}

// K2: counts of chunk c's records in chunk cc, one CTA per ordered pair
// (c, cc != c) so the whole GPU shares the O(n * nchunks * log kChunk)
// searches.  Thread t owns records t, t + 256, ... of chunk c (striped: the
// lanes of a warp search nearby words of the other chunk's high key words,
// which stay L1-resident); kChunkItems fixed-depth branchless binary searches
// run in lock-step (ILP) on the high 32 key bits and fall back to the full
// (key, index) order only when high words tie.  The counts are added to the
// record's rank with integer atomics (exact, so the result is deterministic).
template <int kChunkThreads, int kChunkItems>
__global__ void __launch_bounds__(kChunkThreads)
rank_count_kernel(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ khi,
                  const uint32_t *__restrict__ idx, int *__restrict__ rank)
{
    pdl_wait();  // krcv_pdl.cuh
    constexpr int kChunk = kChunkThreads * kChunkItems;
    const int c = blockIdx.x, cc = blockIdx.y;
    if (c == cc) return;
    const int t = threadIdx.x;
    const uint32_t *ch = khi + (size_t)cc * kChunk;
    const uint64_t *ck = keys + (size_t)cc * kChunk;
    const uint32_t *ci = idx + (size_t)cc * kChunk;
    uint64_t k[kChunkItems];
    uint32_t v[kChunkItems], kh[kChunkItems];
    int pos[kChunkItems];
#pragma unroll
    for (int q = 0; q < kChunkItems; q++) {
        const int g = c * kChunk + t + q * kChunkThreads;
        k[q] = keys[g];
        v[q] = idx[g];
        kh[q] = (uint32_t)(k[q] >> 32);
        pos[q] = 0;
    }
    // pos = #{records of cc that are (key, idx)-less}; invariant: [0, pos) less
#pragma unroll
    for (int half = kChunk / 2; half > 0; half >>= 1) {
#pragma unroll
        for (int q = 0; q < kChunkItems; q++) {
            const int p = pos[q] + half - 1;
            const uint32_t hp = __ldg(ch + p);
            bool less = hp < kh[q];
            if (hp == kh[q]) {  // rare: compare the full order
                const uint64_t kp = __ldg(ck + p);
                less = kp < k[q] || (kp == k[q] && __ldg(ci + p) < v[q]);
            }
            pos[q] += less ? half : 0;
        }
    }
#pragma unroll
    for (int q = 0; q < kChunkItems; q++) {
        const int p = pos[q];  // <= kChunk - 1
        const uint32_t hp = __ldg(ch + p);
        bool less = hp < kh[q];
        if (hp == kh[q]) {
            const uint64_t kp = __ldg(ck + p);
            less = kp < k[q] || (kp == k[q] && __ldg(ci + p) < v[q]);
        }
        if (v[q] != 0xffffffffu) atomicAdd(rank + c * kChunk + t + q * kChunkThreads, p + (less ? 1 : 0));
    }
}

// K3: scatter (x, y) to the sorted positions; sentinels; sweep counter reset.
__global__ void __launch_bounds__(256)
rank_scatter_kernel(const uint32_t *__restrict__ idx, const int *__restrict__ rank, int n, int npad,
                    const double *__restrict__ x, const double *__restrict__ y, double2 *__restrict__ xy,
                    uint32_t *__restrict__ perm, int *__restrict__ tile_counter)
{
    pdl_wait();  // krcv_pdl.cuh
    const int g = blockIdx.x * blockDim.x + threadIdx.x;
    if (g < kPad) {
        xy[-1 - g] = make_double2(-INFINITY, 0.0);
        xy[n + g] = make_double2(INFINITY, 0.0);
    }
    if (g == 0) *tile_counter = 0;
    if (g >= npad) return;
    const uint32_t i = idx[g];
    if (i < (uint32_t)n) {
        const int r = rank[g];
        xy[r] = make_double2(x[i], y[i]);
        perm[r] = i;  // sorted position -> original index (histogram path's self test)
    }
}

// ---------------------------------------------------------------------------
// Large-n sort on a 32-bit quantised key (a2 for n > kRankSortMaxN).  The
// 64-bit order-preserving keys of x are reduced to q = (key - kmin) >> s with
// s = max(0, bitlen(kmax - kmin) - 32), a monotone map onto 32 bits, so a
// stable 4-pass radix sort of (q, index) orders the records by x up to runs
// of equal q; each such run (x values within 2^s key units of each other --
// a few records at most for real data) is then put in exact (key, index)
// order by insertion sort (already-sorted runs, e.g. duplicates, cost one
// comparison per record).  Half the passes of the 64-bit sort, the same
// total order (stable by original index).
// ---------------------------------------------------------------------------
// pack: validation counters (as pack_kernel) and the key range, kept as
// atomicMax of the complemented minimum / of the maximum (zero-initialised
// by the call's status memset)
__global__ void pack_range_kernel(const double *__restrict__ x, const double *__restrict__ y, int n,
                                  const double *__restrict__ h, int m, unsigned *__restrict__ status,
                                  unsigned long long *__restrict__ kmin_c, unsigned long long *__restrict__ kmax)
{
    const int stride = gridDim.x * blockDim.x;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned bad = 0, gbad = 0;
    unsigned long long lo = ~0ull, hi = 0ull;
    for (int i = tid; i < n; i += stride) {
        const double xv = x[i], yv = y[i];
        bad += (!isfinite(xv) || !isfinite(yv)) ? 1u : 0u;
        const unsigned long long k = order_key(xv);
        lo = k < lo ? k : lo;
        hi = k > hi ? k : hi;
    }
    for (int b = tid; b < m; b += stride) {
        const double hb = h[b];
        gbad += (!isfinite(hb) || !(hb > 0.0) || (b > 0 && hb < h[b - 1])) ? 1u : 0u;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long a = __shfl_xor_sync(0xffffffffu, lo, o), c = __shfl_xor_sync(0xffffffffu, hi, o);
        lo = a < lo ? a : lo;
        hi = c > hi ? c : hi;
    }
    // one atomic per CTA (per warp, thousands of same-address atomics
    // serialised in L2: 11 us at n = 200,000, profiles/r02/r02ad_*)
    __shared__ unsigned long long slo[32], shi[32];
    __shared__ unsigned sbad[32], sgbad[32];
    const int w = threadIdx.x >> 5, nw = (blockDim.x + 31) >> 5;
    if ((threadIdx.x & 31) == 0) {
        slo[w] = lo;
        shi[w] = hi;
    }
    bad = __reduce_add_sync(0xffffffffu, bad);
    gbad = __reduce_add_sync(0xffffffffu, gbad);
    if ((threadIdx.x & 31) == 0) {
        sbad[w] = bad;
        sgbad[w] = gbad;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int q = 1; q < nw; q++) {
            lo = slo[q] < lo ? slo[q] : lo;
            hi = shi[q] > hi ? shi[q] : hi;
            bad += sbad[q];
            gbad += sgbad[q];
        }
        if (hi >= lo) {
            atomicMax(kmin_c, ~lo);
            atomicMax(kmax, hi);
        }
        if (bad) atomicAdd(&status[1], bad);
        if (gbad) atomicAdd(&status[0], gbad);
    }
}

__device__ __forceinline__ int q32_shift(unsigned long long kmin, unsigned long long kmax)
{
    const unsigned long long r = kmax - kmin;
    const int bits = r ? 64 - __clzll((long long)r) : 0;
    return bits > 32 ? bits - 32 : 0;
}

__global__ void quant_kernel(const double *__restrict__ x, int n, const unsigned long long *__restrict__ kmin_c,
                             const unsigned long long *__restrict__ kmax, uint32_t *__restrict__ q,
                             uint32_t *__restrict__ idx)
{
    pdl_wait();  // krcv_pdl.cuh
    const unsigned long long lo = ~*kmin_c, hi = *kmax;
    const int s = q32_shift(lo, hi);
    const int stride = gridDim.x * blockDim.x;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        q[i] = (uint32_t)((order_key(x[i]) - lo) >> s);
        idx[i] = (uint32_t)i;
    }
}

// exact (key, index) order inside every run of equal q (sorted positions)
__global__ void q32_fixup_kernel(const double *__restrict__ x, int n, const uint32_t *__restrict__ q,
                                 uint32_t *__restrict__ idx)
{
    pdl_wait();  // krcv_pdl.cuh
    const int stride = gridDim.x * blockDim.x;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
        const uint32_t qi = q[i];
        if ((i > 0 && q[i - 1] == qi) || i + 1 >= n || q[i + 1] != qi) continue;  // not the start of a run >= 2
        int e = i + 2;
        while (e < n && q[e] == qi) e++;
        for (int a = i + 1; a < e; a++) {  // insertion sort by (key, index); stable input order is index order
            const uint32_t v = idx[a];
            const unsigned long long kv = order_key(x[v]);
            int b = a - 1;
            while (b >= i) {
                const uint32_t u = idx[b];
                const unsigned long long ku = order_key(x[u]);
                if (ku < kv || (ku == kv && u < v)) break;
                idx[b + 1] = u;
                b--;
            }
            idx[b + 1] = v;
        }
    }
}

}  // namespace krcv
