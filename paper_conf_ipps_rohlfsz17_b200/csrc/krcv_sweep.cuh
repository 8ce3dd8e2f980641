// krcv_sweep.cuh -- the hot loop (SURVEY.md §8 rows a3 + a4), sm_100a, fp64.
//
// PAPER.md §III P@14010-14984 and §IV.B P@21154-22104: for every row i the
// neighbours are visited in increasing |X_i - X_l|; the running sums for
// bandwidth h_b are "copied" to h_{b+1} and extended with the additional
// neighbours.  Here the ordering comes from ONE global sort (a2): in the
// sorted array row i's right neighbours i+1, i+2, ... and left neighbours
// i-1, i-2, ... are each already in increasing distance, so the per-row sort
// of the paper (P@20542) disappears and the running sums live in registers.
//
// Work decomposition:
//   * a warp owns a tile of RPW = 32/G consecutive sorted rows;
//   * the G lanes of a row split BOTH sides' neighbour streams by residue
//     class (lane k takes j = i+1+k, i+1+k+G, ...; monotone per class, so
//     "4th element inside => all four inside" still holds);
//   * per iteration a lane consumes a quad on the right AND a quad on the
//     left (two independent load/accumulate chains for ILP);
//   * bandwidths ascend warp-uniformly; at each h_b the G lanes combine
//     their sums with a shuffle butterfly and every lane evaluates the LOO
//     estimate (a4) -- lane k==0 contributes e^2;
//   * the per-(tile, b) sums of M e^2 and M are written once by lane 0.
//   * tiles are handed out dynamically (atomic counter) but written to
//     tile-indexed slots, so results are bit-reproducible.
//
// The sorted (x, y) array carries +/-inf sentinels (kPad records on each
// side) so quads never bounds-check: d = +inf is outside every window.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "krcv.h"

namespace krcv {

constexpr int kPad = 32;            // sentinel records on each side of xy
constexpr int kSweepWarps = 4;      // warps per CTA
constexpr int kSweepThreads = kSweepWarps * 32;

template <int KERN>
__device__ __forceinline__ bool inside(double d, double h)
{
    // Reading Q1: open window for Epanechnikov / triangular, closed for uniform.
    return KERN == KR_UNIFORM ? (d <= h) : (d < h);
}

// Running sums (reading Q3).  Epanechnikov: sum y, sum d^2, sum y d^2.
// Triangular: sum y, sum d, sum y d.  Uniform: sum y.  The count comes from
// the pointers.
struct Sums {
    double sy, s1, sy1;
};

template <int KERN>
__device__ __forceinline__ void acc(Sums &s, double yv, double d)
{
    s.sy += yv;
    if (KERN == KR_EPANECHNIKOV) {
        const double d2 = d * d;
        s.s1 += d2;
        s.sy1 = fma(yv, d2, s.sy1);
    } else if (KERN == KR_TRIANGULAR) {
        s.s1 += d;
        s.sy1 = fma(yv, d, s.sy1);
    }
}

// Consume one quad of a side.  p = next candidate index of this lane's
// residue class, step = +G (right) or -G (left).  Elements alternate between
// two accumulator sets (sa: 0, 2; sb: 1, 3) to halve the dependency chains.
// Returns true if the side may still have in-window elements for this
// bandwidth.
template <int KERN, int G, bool RIGHT>
__device__ __forceinline__ bool quad(int &p, int &cnt, Sums &sa, Sums &sb, double xi, double h,
                                     const double2 &v0, const double2 &v1, const double2 &v2,
                                     const double2 &v3)
{
    const double d0 = RIGHT ? v0.x - xi : xi - v0.x;
    const double d1 = RIGHT ? v1.x - xi : xi - v1.x;
    const double d2 = RIGHT ? v2.x - xi : xi - v2.x;
    const double d3 = RIGHT ? v3.x - xi : xi - v3.x;
    constexpr int step = RIGHT ? G : -G;
    if (inside<KERN>(d3, h)) {  // monotone: all four inside
        acc<KERN>(sa, v0.y, d0);
        acc<KERN>(sb, v1.y, d1);
        acc<KERN>(sa, v2.y, d2);
        acc<KERN>(sb, v3.y, d3);
        p += 4 * step;
        cnt += 4;
        return true;
    }
    // partial quad: the inside elements form a prefix
    if (inside<KERN>(d0, h)) {
        acc<KERN>(sa, v0.y, d0);
        p += step;
        cnt += 1;
        if (inside<KERN>(d1, h)) {
            acc<KERN>(sb, v1.y, d1);
            p += step;
            cnt += 1;
            if (inside<KERN>(d2, h)) {
                acc<KERN>(sa, v2.y, d2);
                p += step;
                cnt += 1;
            }
        }
    }
    return false;
}

template <int G>
__device__ __forceinline__ double group_sum(double v)
{
#pragma unroll
    for (int o = 1; o < G; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

template <int G>
__device__ __forceinline__ int group_sum_i(int v)
{
#pragma unroll
    for (int o = 1; o < G; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

__device__ __forceinline__ double warp_sum(double v)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// xy points at the first real record; xy[-kPad .. -1] = (-inf, 0) and
// xy[n .. n+kPad-1] = (+inf, 0).
template <int KERN, int G>
__global__ void __launch_bounds__(kSweepThreads)
sweep_kernel(const double2 *__restrict__ xy, int n, const double *__restrict__ hg, int m,
             int row_lo, int row_hi, int ntiles, double *__restrict__ tileS, uint8_t *__restrict__ tileN,
             int *__restrict__ tile_counter)
{
    constexpr int RPW = 32 / G;  // rows per warp tile
    const int lane = threadIdx.x & 31;
    const int slot = lane / G;   // row within the tile
    const int k = lane % G;      // residue class within the row's streams
    // k==0 lanes carry the row's e^2 / M into the warp reductions
    const unsigned lead_mask = (G == 1) ? 0xffffffffu : (G == 2 ? 0x55555555u : (G == 4 ? 0x11111111u : 0x01010101u));

    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) return;  // warp-uniform

        const int i = row_lo + tile * RPW + slot;
        const bool valid = i < row_hi;
        double xi = 0.0, yi = 0.0;
        if (valid) {
            const double2 v = xy[i];
            xi = v.x;
            yi = v.y;
        }
        int R = i + 1 + k, L = i - 1 - k;  // this lane's next right / left candidates
        int cR = 0, cL = 0;                // this lane's in-window counts
        Sums sRa{0.0, 0.0, 0.0}, sRb{0.0, 0.0, 0.0}, sLa{0.0, 0.0, 0.0}, sLb{0.0, 0.0, 0.0};

        for (int b = 0; b < m; b++) {
            const double h = __ldg(hg + b);
            bool rgo = valid, lgo = valid;
            while (rgo || lgo) {
                double2 a0, a1, a2, a3, c0, c1, c2, c3;
                if (rgo) {
                    a0 = xy[R];
                    a1 = xy[R + G];
                    a2 = xy[R + 2 * G];
                    a3 = xy[R + 3 * G];
                }
                if (lgo) {
                    c0 = xy[L];
                    c1 = xy[L - G];
                    c2 = xy[L - 2 * G];
                    c3 = xy[L - 3 * G];
                }
                if (rgo) rgo = quad<KERN, G, true>(R, cR, sRa, sRb, xi, h, a0, a1, a2, a3);
                if (lgo) lgo = quad<KERN, G, false>(L, cL, sLa, sLb, xi, h, c0, c1, c2, c3);
            }

            // ---- a4: combine the row's G lanes, LOO estimate, squared error
            const int cRt = group_sum_i<G>(cR);
            const int cLt = group_sum_i<G>(cL);
            const double sy = group_sum<G>((sRa.sy + sRb.sy) + (sLa.sy + sLb.sy));
            double s1 = 0.0, sy1 = 0.0;
            if (KERN != KR_UNIFORM) {
                s1 = group_sum<G>((sRa.s1 + sRb.s1) + (sLa.s1 + sLb.s1));
                sy1 = group_sum<G>((sRa.sy1 + sRb.sy1) + (sLa.sy1 + sLb.sy1));
            }
            const int c = cRt + cLt;
            const bool M = valid && c > 0;  // reading Q6
            double e2 = 0.0;
            if (M) {
                double g;
                if (KERN == KR_UNIFORM) {
                    g = sy / (double)c;
                } else {
                    // Eq.(2)-(3) with 0.75 and 1/h^2 cancelled (reading Q5)
                    const double hk = (KERN == KR_EPANECHNIKOV) ? h * h : h;
                    double num = fma(hk, sy, -sy1);
                    double den = fma(hk, (double)c, -s1);
                    // Reading Q14: if the decomposition has cancelled,
                    // recompute directly over the contiguous window
                    // [i - cLt, i + cRt] \ {i} with exact factors.
                    if (!(den >= 0x1p-20 * hk * (double)c)) {
                        num = 0.0;
                        den = 0.0;
                        for (int q = i - cLt; q <= i + cRt; q++) {
                            if (q == i) continue;
                            const double2 v = xy[q];
                            const double d = fabs(v.x - xi);
                            const double w = (KERN == KR_EPANECHNIKOV) ? (h - d) * (h + d) : (h - d);
                            num = fma(v.y, w, num);
                            den += w;
                        }
                    }
                    g = num / den;
                }
                const double e = yi - g;
                e2 = (k == 0) ? e * e : 0.0;
            }
            // ---- a5 (warp level): fixed shuffle tree over the tile's rows
            e2 = warp_sum(e2);
            const unsigned ball = __ballot_sync(0xffffffffu, M) & lead_mask;
            if (lane == 0) {
                tileS[(size_t)b * ntiles + tile] = e2;
                tileN[(size_t)b * ntiles + tile] = (uint8_t)__popc(ball);
            }
        }
    }
}

}  // namespace krcv
