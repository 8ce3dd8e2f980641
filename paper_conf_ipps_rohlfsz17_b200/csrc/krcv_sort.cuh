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
//      entries, and radix-sorts the chunk in registers/shared memory
//      (cub::BlockRadixSort, stable, so ties stay in index order);
//   K2 rank_scatter_kernel: every record's final position is its position in
//      its chunk plus, for every other chunk, the number of records that
//      compare less (branchless binary search); it writes (x, y) straight to
//      that position of the sorted array -- no merge passes, no separate
//      gather.  (key, index) pairs are unique, so the order is total and
//      identical to a stable sort by x.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include <cub/block/block_radix_sort.cuh>

#include "krcv_sweep.cuh"

namespace krcv {

constexpr int kChunkThreads = 256;
constexpr int kChunkItems = 8;
constexpr int kChunk = kChunkThreads * kChunkItems;  // 2048 records per CTA in K1
constexpr int64_t kRankSortMaxN = 64 * kChunk;     // 131072: <= 63 searches per record

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

__global__ void __launch_bounds__(kChunkThreads)
chunk_sort_kernel(const double *__restrict__ x, const double *__restrict__ y, int n,
                  const double *__restrict__ h, int m, uint64_t *__restrict__ keys,
                  uint32_t *__restrict__ idx, unsigned *__restrict__ status)
{
    using BRS = cub::BlockRadixSort<uint64_t, kChunkThreads, kChunkItems, uint32_t, 6>;
    __shared__ typename BRS::TempStorage ts;
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
    BRS(ts).Sort(k, v);  // stable LSD radix: equal keys keep index order
#pragma unroll
    for (int q = 0; q < kChunkItems; q++) {
        keys[base + threadIdx.x * kChunkItems + q] = k[q];
        idx[base + threadIdx.x * kChunkItems + q] = v[q];
    }
}

constexpr int kSearchBatch = 8;      // binary searches advanced in lock-step (ILP)
constexpr int kRankThreads = 256;    // a CTA ranks 256 consecutive records of one chunk
constexpr int kMaxChunks = (int)(kRankSortMaxN / kChunk);

// Branchless count of records < (k, i) in the sorted range [lo, lo + len) of
// the chunked arrays, for kSearchBatch chunks at once.
__device__ __forceinline__ bool rec_less(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ idx,
                                         int p, uint64_t k, uint32_t i)
{
    const uint64_t kp = keys[p];
    return kp < k || (kp == k && idx[p] < i);  // idx only read on key ties
}

__global__ void __launch_bounds__(kRankThreads)
rank_scatter_kernel(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ idx, int n, int nchunks,
                    const double *__restrict__ x, const double *__restrict__ y, double2 *__restrict__ xy,
                    int *__restrict__ tile_counter)
{
    __shared__ int s_lo[kMaxChunks], s_len[kMaxChunks];
    const int g0 = blockIdx.x * kRankThreads;  // first record of this CTA (sorted within chunk c)
    const int g = g0 + threadIdx.x;
    const int c = g0 / kChunk;
    if (g < kPad && blockIdx.x == 0) {
        xy[-1 - g] = make_double2(-INFINITY, 0.0);
        xy[n + g] = make_double2(INFINITY, 0.0);
    }
    if (g == 0) *tile_counter = 0;
    // 1) For every other chunk, bracket where this CTA's records fall: the
    //    counts of its first and last record (2 full searches per chunk, one
    //    thread each).  Every record's count then lies in that bracket, which
    //    the whole CTA searches next -- a small, L1-resident range.
    {
        const int t = threadIdx.x;
        if (t < 2 * nchunks) {
            const int cc = t >> 1;
            const int gq = (t & 1) ? g0 + kRankThreads - 1 : g0;
            const uint64_t kq = keys[gq];
            const uint32_t iq = idx[gq];
            int base = 0;
#pragma unroll
            for (int half = kChunk / 2; half > 0; half >>= 1)
                if (rec_less(keys, idx, cc * kChunk + base + half - 1, kq, iq)) base += half;
            base += rec_less(keys, idx, cc * kChunk + base, kq, iq) ? 1 : 0;
            if (t & 1) s_len[cc] = base;  // count for the last record (upper end)
            else s_lo[cc] = base;
        }
    }
    __syncthreads();
    if (g >= nchunks * kChunk) return;
    const uint32_t i = idx[g];
    if (i >= (uint32_t)n) return;  // padding
    const uint64_t k = keys[g];
    int rank = g - c * kChunk;
    // 2) count within [lo, hi] of each other chunk; kSearchBatch searches in
    //    lock-step; ranges are short, so fixed-depth searches over pow2 spans.
    for (int c0 = 0; c0 < nchunks; c0 += kSearchBatch) {
        int basev[kSearchBatch], hiv[kSearchBatch];
#pragma unroll
        for (int j = 0; j < kSearchBatch; j++) {
            const int cc = min(c0 + j, nchunks - 1);
            basev[j] = s_lo[cc];        // count >= this
            hiv[j] = s_len[cc];         // count <= this
        }
        // widest bracket of the batch decides the depth (warp-uniform loop)
        int span = 0;
#pragma unroll
        for (int j = 0; j < kSearchBatch; j++) span = max(span, hiv[j] - basev[j]);
        int step = 1;
        while (step <= span) step <<= 1;
        for (step >>= 1; step > 0; step >>= 1) {
#pragma unroll
            for (int j = 0; j < kSearchBatch; j++) {
                const int cc = min(c0 + j, nchunks - 1);
                const int q = basev[j] + step;  // candidate count
                if (q <= hiv[j] && rec_less(keys, idx, cc * kChunk + q - 1, k, i)) basev[j] = q;
            }
        }
#pragma unroll
        for (int j = 0; j < kSearchBatch; j++) {
            const int cc = c0 + j;
            if (cc < nchunks && cc != c) rank += basev[j];
        }
    }
    xy[rank] = make_double2(x[i], y[i]);
}

}  // namespace krcv
