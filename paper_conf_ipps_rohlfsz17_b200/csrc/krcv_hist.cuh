// krcv_hist.cuh -- the bucket-by-bandwidth histogram ordering (SURVEY.md
// §7.1 design "H", ablation N8; BASELINE.json north_star: "a
// bucket-by-bandwidth shared-memory histogram followed by a warp-shuffle
// scan, which gives the same sums without a full sort").
//
// The paper orders each row's n-1 distances with a private sort so that one
// pass of running sums serves every bandwidth (§III P@14377-14984, §IV.B
// P@20542-22104).  The running sums at h_b only need the neighbours grouped
// by the first bandwidth whose window holds them, not their order inside a
// group, so here:
//   1. every neighbour j != i (streamed in the caller's original order -- no
//      sort of the neighbours) gets its bucket b(j) = min{ b : d_ij in the
//      window of h_b } (reading Q1's exact binary64 predicate, found by a
//      branchless binary search of the grid in shared memory; b = m if j is
//      outside every window);
//   2. c, sum y, sum d^2, sum y d^2 (uniform: c, sum y; triangular: c, sum y,
//      sum d, sum y d) are added into the row's shared-memory histogram slot
//      b with shared-memory atomics (fp64 adds are CAS loops on sm_100a);
//   3. a warp-shuffle inclusive scan over the buckets turns the histogram
//      into the running sums of every bandwidth at once, and each lane emits
//      the LOO estimate, M and the squared error of its buckets (the same
//      formulas and reading-Q14 guard as the sweep).
// The rows of a shard are the sorted-order rows (so shards mean the same as
// on the other paths); `perm` maps a sorted row to its original index, which
// the neighbour stream skips (LOO, Eq.(2) l != i, reading Q8).
//
// The atomics make the summation order timing-dependent: results agree with
// the other paths to rounding (~1e-15), not bit for bit.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "krcv.h"
#include "krcv_sweep.cuh"

namespace krcv {

constexpr int kHistMaxWarps = 8;

// Shared-memory bytes of one warp's slice: int count + 3 fp64 sums per
// bucket, plus the warp's per-bandwidth accumulators over its 32 rows.
__host__ __device__ constexpr size_t hist_warp_bytes(int m)
{
    return (size_t)m * (sizeof(int) + 3 * sizeof(double)) + (size_t)m * (sizeof(double) + sizeof(int));
}

__host__ __device__ constexpr size_t hist_smem_bytes(int m, int warps)
{
    return (size_t)m * sizeof(double) + (size_t)warps * hist_warp_bytes(m);
}

// First bucket whose window holds distance d (m if none): the count of grid
// points h_k with d outside the window of h_k (monotone: outside for small h).
template <int KERN>
__device__ __forceinline__ int hist_bucket(const double *__restrict__ hs, int m, int p2, double d)
{
    int b = 0;
    for (int s = p2; s > 0; s >>= 1) {
        const int t = b + s;
        if (t <= m && !inside<KERN>(d, hs[t - 1])) b = t;
    }
    return b;
}

template <int KERN>
__global__ void __launch_bounds__(kHistMaxWarps * 32)
hist_kernel(const double *__restrict__ x, const double *__restrict__ y, const uint32_t *__restrict__ perm,
            const double2 *__restrict__ xy, const double *__restrict__ hg, int m, int n, int row_lo, int row_hi,
            int ntiles, double *__restrict__ tileS, uint8_t *__restrict__ tileN, int *__restrict__ tile_counter)
{
    extern __shared__ __align__(16) unsigned char smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    double *hs = reinterpret_cast<double *>(smem);
    unsigned char *base = smem + (size_t)m * sizeof(double) + (size_t)warp * hist_warp_bytes(m);
    double *hy = reinterpret_cast<double *>(base);   // sum y
    double *h2 = hy + m;                             // sum d^2 (triangular: sum d)
    double *hy2 = h2 + m;                            // sum y d^2 (triangular: sum y d)
    double *accS = hy2 + m;                          // per-bandwidth sum of M e^2 over the warp's rows
    int *hc = reinterpret_cast<int *>(accS + m);     // count
    int *accN = hc + m;                              // per-bandwidth sum of M
    for (int b = threadIdx.x; b < m; b += blockDim.x) hs[b] = hg[b];
    __syncthreads();
    int p2 = 1;
    while (p2 * 2 <= m) p2 *= 2;
    // one 32-row tile per CTA iteration: warp w takes rows r0 + w, r0 + w + nw, ...
    __shared__ int task_s;
    for (;;) {
        if (threadIdx.x == 0) task_s = atomicAdd(tile_counter, 1);
        __syncthreads();
        const int task = task_s;
        __syncthreads();
        if (task >= ntiles) return;  // CTA-uniform
        for (int b = lane; b < m; b += 32) {
            accS[b] = 0.0;
            accN[b] = 0;
        }
        const int r0 = row_lo + task * 32;
        const int r1 = min(row_hi, r0 + 32);
        for (int r = r0 + warp; r < r1; r += nw) {
            for (int b = lane; b < m; b += 32) {
                hc[b] = 0;
                hy[b] = 0.0;
                h2[b] = 0.0;
                hy2[b] = 0.0;
            }
            __syncwarp();
            const double2 me = xy[r];
            const double xi = me.x, yi = me.y;
            const uint32_t self = perm[r];
            // 1 + 2: bucket every neighbour, shared-memory atomics
            for (int j = lane; j < n; j += 32) {
                if ((uint32_t)j == self) continue;
                const double d = fabs(x[j] - xi);
                const int b = hist_bucket<KERN>(hs, m, p2, d);
                if (b >= m) continue;
                const double yj = y[j];
                atomicAdd(&hc[b], 1);
                atomicAdd(&hy[b], yj);
                if (KERN == KR_EPANECHNIKOV) {
                    const double d2 = d * d;
                    atomicAdd(&h2[b], d2);
                    atomicAdd(&hy2[b], yj * d2);
                } else if (KERN == KR_TRIANGULAR) {
                    atomicAdd(&h2[b], d);
                    atomicAdd(&hy2[b], yj * d);
                }
            }
            __syncwarp();
            // 3: warp-shuffle inclusive scan over buckets, emit per bucket
            int cc = 0;
            double cy = 0.0, c2 = 0.0, cy2 = 0.0;
            for (int b0 = 0; b0 < m; b0 += 32) {
                const int b = b0 + lane;
                int vc = 0;
                double vy = 0.0, v2 = 0.0, vy2 = 0.0;
                if (b < m) {
                    vc = hc[b];
                    vy = hy[b];
                    v2 = h2[b];
                    vy2 = hy2[b];
                }
#pragma unroll
                for (int s = 1; s < 32; s <<= 1) {
                    const int tc = __shfl_up_sync(0xffffffffu, vc, s);
                    const double ty = __shfl_up_sync(0xffffffffu, vy, s);
                    const double t2 = __shfl_up_sync(0xffffffffu, v2, s);
                    const double ty2 = __shfl_up_sync(0xffffffffu, vy2, s);
                    if (lane >= s) {
                        vc += tc;
                        vy += ty;
                        v2 += t2;
                        vy2 += ty2;
                    }
                }
                vc += cc;
                vy += cy;
                v2 += c2;
                vy2 += cy2;
                cc = __shfl_sync(0xffffffffu, vc, 31);
                cy = __shfl_sync(0xffffffffu, vy, 31);
                c2 = __shfl_sync(0xffffffffu, v2, 31);
                cy2 = __shfl_sync(0xffffffffu, vy2, 31);
                if (b < m && vc > 0) {  // reading Q6: M = [c >= 1]
                    const double h = hs[b];
                    double g;
                    if (KERN == KR_UNIFORM) {
                        g = vy / (double)vc;
                    } else {
                        const double hk = KERN == KR_EPANECHNIKOV ? h * h : h;
                        double num = fma(hk, vy, -vy2);
                        double den = fma(hk, (double)vc, -v2);
                        if (!(den >= 0x1p-20 * hk * (double)vc)) {  // reading Q14: direct recompute
                            num = 0.0;
                            den = 0.0;
                            for (int j = 0; j < n; j++) {
                                if ((uint32_t)j == self) continue;
                                const double d = fabs(x[j] - xi);
                                if (!inside<KERN>(d, h)) continue;
                                const double w = KERN == KR_EPANECHNIKOV ? (h - d) * (h + d) : (h - d);
                                num = fma(y[j], w, num);
                                den += w;
                            }
                        }
                        g = num / den;
                    }
                    const double e = yi - g;
                    accS[b] = fma(e, e, accS[b]);
                    accN[b] += 1;
                }
            }
            __syncwarp();
        }
        __syncthreads();
        // the tile's per-bandwidth sums: warps' accumulators in a fixed order
        for (int b = threadIdx.x; b < m; b += blockDim.x) {
            double sS = 0.0;
            int sN = 0;
            for (int w2 = 0; w2 < nw; w2++) {
                const unsigned char *bw = smem + (size_t)m * sizeof(double) + (size_t)w2 * hist_warp_bytes(m);
                const double *aS = reinterpret_cast<const double *>(bw) + 3 * m;
                const int *aN = reinterpret_cast<const int *>(aS + m) + m;
                sS += aS[b];
                sN += aN[b];
            }
            tileS[(size_t)b * ntiles + task] = sS;
            tileN[(size_t)b * ntiles + task] = (uint8_t)sN;
        }
    }
}

}  // namespace krcv
