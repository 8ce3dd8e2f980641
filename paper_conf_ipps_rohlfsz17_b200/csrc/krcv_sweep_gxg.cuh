// krcv_sweep_gxg.cuh -- "G x G" variant of the sweep (rows a3 + a4).
//
// Same method as krcv_sweep.cuh (§III P@14010-14984: nested windows,
// running sums carried from h_b to h_{b+1}); different work decomposition:
//
//   * a group of G lanes owns G ADJACENT sorted rows i0 .. i0+G-1;
//   * lane k of the group visits the neighbours j with j = k (mod G)
//     (absolute residue class) for ALL G rows at once: every element it
//     loads (16 B) feeds G pairs, so L1->register traffic per pair is 16/G B
//     (the split variant moves 16 B per pair; ncu showed that writeback path,
//     128 B/clk/SM, bounding it);
//   * the rows' windows differ only by the few points between x_i0 + h and
//     x_{i0+G-1} + h, so one shared stream per side serves all rows; each
//     (row, element) slot is taken iff the element is inside that row's
//     window and not already counted (index predicate);
//   * at each h_b a reduce-scatter over the G lanes leaves lane k with the
//     totals of row i0+k, which it alone turns into the LOO estimate (a4):
//     no redundant epilogues;
//   * warp = 32 consecutive rows; tiles handed out by an atomic counter,
//     written to tile-indexed slots (bit-reproducible).
#pragma once

#include "krcv_sweep.cuh"

namespace krcv {

// Reduce-scatter of v[0..G-1] over the G lanes of a group (xor butterfly,
// halving): lane k returns sum over the group of v[k].  G-1 shuffles.
template <int G, typename T>
__device__ __forceinline__ T reduce_scatter(const T (&v)[G], int k)
{
    if constexpr (G == 1) {
        return v[0];
    } else if constexpr (G == 2) {
        const T keep = (k & 1) ? v[1] : v[0];
        const T send = (k & 1) ? v[0] : v[1];
        return keep + __shfl_xor_sync(0xffffffffu, send, 1);
    } else {
        const bool hi = (k & 2) != 0;
        T a = hi ? v[2] : v[0];
        T b = hi ? v[3] : v[1];
        const T sa = hi ? v[0] : v[2];
        const T sb = hi ? v[1] : v[3];
        a += __shfl_xor_sync(0xffffffffu, sa, 2);
        b += __shfl_xor_sync(0xffffffffu, sb, 2);
        const T keep = (k & 1) ? b : a;
        const T send = (k & 1) ? a : b;
        return keep + __shfl_xor_sync(0xffffffffu, send, 1);
    }
}

template <int KERN, int G>
__global__ void __launch_bounds__(kSweepThreads)
sweep_gxg_kernel(const double2 *__restrict__ xy, int n, const double *__restrict__ hg, int m,
                 int row_lo, int row_hi, int ntiles, double *__restrict__ tileS, uint8_t *__restrict__ tileN,
                 int *__restrict__ tile_counter)
{
    const int lane = threadIdx.x & 31;
    const int k = lane & (G - 1);  // residue class of this lane
    const int grp = lane / G;

    for (;;) {
        int tile = 0;
        if (lane == 0) tile = atomicAdd(tile_counter, 1);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= ntiles) return;  // warp-uniform

        const int i0 = row_lo + tile * 32 + grp * G;
        const bool gvalid = i0 < row_hi;
        // Rows of the group.  Rows past the shard end are clamped to the last
        // valid row (identical work, discarded) so x stays non-decreasing.
        double xr[G], yr[G];
        int nx[G], pv[G], first_n[G], first_p[G];  // next right / prev left candidate in class k
#pragma unroll
        for (int r = 0; r < G; r++) {
            const int ir = min(i0 + r, row_hi - 1);
            const double2 v = gvalid ? xy[ir] : make_double2(0.0, 0.0);
            xr[r] = v.x;
            yr[r] = v.y;
            nx[r] = ir + 1 + ((k - ir - 1) & (G - 1));  // first j > ir with j = k (mod G)
            pv[r] = ir - 1 - ((ir - 1 - k) & (G - 1));  // last j < ir with j = k (mod G)
            first_n[r] = nx[r];
            first_p[r] = pv[r];
        }
        Sums sR[G], sL[G];
#pragma unroll
        for (int r = 0; r < G; r++) {
            sR[r] = Sums{0.0, 0.0, 0.0};
            sL[r] = Sums{0.0, 0.0, 0.0};
        }

        for (int b = 0; b < m; b++) {
            const double h = __ldg(hg + b);
            // Right: row 0 lags (largest d), row G-1 reaches farthest.
            // Left: row G-1 lags, row 0 reaches farthest.
            int pR = nx[0], pL = pv[G - 1];
            bool rgo = gvalid, lgo = gvalid;
            while (rgo || lgo) {
                double2 a[4], c[4];
                if (rgo) {
#pragma unroll
                    for (int q = 0; q < 4; q++) a[q] = xy[pR + q * G];
                }
                if (lgo) {
#pragma unroll
                    for (int q = 0; q < 4; q++) c[q] = xy[pL - q * G];
                }
                if (rgo) {
                    bool lead_in = false;
#pragma unroll
                    for (int r = 0; r < G; r++) {
                        int cnt = 0;
#pragma unroll
                        for (int q = 0; q < 4; q++) {
                            const double d = a[q].x - xr[r];
                            const bool in = inside<KERN>(d, h);
                            cnt += in ? 1 : 0;
                            if (in && pR + q * G >= nx[r]) acc<KERN>(sR[r], a[q].y, d);
                            if (r == G - 1 && q == 3) lead_in = in;
                        }
                        // first outside element of row r = pR + cnt*G, but only in
                        // the quad where row r's inside-prefix ends (cnt > 0);
                        // later quads of this bucket lie wholly outside row r.
                        if (cnt) nx[r] = max(nx[r], pR + cnt * G);
                    }
                    pR += 4 * G;
                    rgo = lead_in;
                }
                if (lgo) {
                    bool lead_in = false;
#pragma unroll
                    for (int r = 0; r < G; r++) {
                        int cnt = 0;
#pragma unroll
                        for (int q = 0; q < 4; q++) {
                            const double d = xr[r] - c[q].x;
                            const bool in = inside<KERN>(d, h);
                            cnt += in ? 1 : 0;
                            if (in && pL - q * G <= pv[r]) acc<KERN>(sL[r], c[q].y, d);
                            if (r == 0 && q == 3) lead_in = in;
                        }
                        if (cnt) pv[r] = min(pv[r], pL - cnt * G);
                    }
                    pL -= 4 * G;
                    lgo = lead_in;
                }
            }

            // ---- a4: reduce-scatter -> lane k owns row i0 + k
            int cRv[G], cLv[G];
            double syv[G], s1v[G], sy1v[G];
#pragma unroll
            for (int r = 0; r < G; r++) {
                cRv[r] = (nx[r] - first_n[r]) / G;
                cLv[r] = (first_p[r] - pv[r]) / G;
                syv[r] = sR[r].sy + sL[r].sy;
                s1v[r] = sR[r].s1 + sL[r].s1;
                sy1v[r] = sR[r].sy1 + sL[r].sy1;
            }
            const int cRt = reduce_scatter<G>(cRv, k);
            const int cLt = reduce_scatter<G>(cLv, k);
            const double sy = reduce_scatter<G>(syv, k);
            double s1 = 0.0, sy1 = 0.0;
            if (KERN != KR_UNIFORM) {
                s1 = reduce_scatter<G>(s1v, k);
                sy1 = reduce_scatter<G>(sy1v, k);
            }
            const int i = i0 + k;
            double xi = xr[0], yi = yr[0];
#pragma unroll
            for (int r = 1; r < G; r++)
                if (k == r) {
                    xi = xr[r];
                    yi = yr[r];
                }
            const int c = cRt + cLt;
            const bool M = gvalid && i < row_hi && c > 0;  // reading Q6
            double e2 = 0.0;
            if (M) {
                double g;
                if (KERN == KR_UNIFORM) {
                    g = sy / (double)c;
                } else {
                    const double hk = (KERN == KR_EPANECHNIKOV) ? h * h : h;
                    double num = fma(hk, sy, -sy1);
                    double den = fma(hk, (double)c, -s1);
                    if (!(den >= 0x1p-20 * hk * (double)c)) {  // reading Q14
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
                e2 = e * e;
            }
            e2 = warp_sum(e2);
            const unsigned ball = __ballot_sync(0xffffffffu, M);
            if (lane == 0) {
                tileS[(size_t)b * ntiles + tile] = e2;
                tileN[(size_t)b * ntiles + tile] = (uint8_t)__popc(ball);
            }
        }
    }
}

}  // namespace krcv
