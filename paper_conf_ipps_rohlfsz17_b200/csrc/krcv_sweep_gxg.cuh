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

// Moments of the elements that lie inside ALL G rows' windows, taken about
// x0 = x of the group's first row: u = x_j - x0.  Row r (delta = x_r - x0)
// recovers its own sums exactly in real arithmetic:
//   sum (x_j - x_r)^2     = u2 - 2 delta u1 + delta^2 c
//   sum y_j (x_j - x_r)^2 = y2 - 2 delta y1 + delta^2 y0
// Such elements satisfy |x_j - x_r| < h for every row, so delta < h and the
// shift adds no cancellation beyond a small constant factor.
struct Shared {
    double c, u1, u2, y0, y1, y2;
};

template <int KERN>
__device__ __forceinline__ void sh_add(Shared &s, double yv, double u)
{
    s.c += 1.0;
    s.y0 += yv;
    if (KERN != KR_UNIFORM) {
        s.u1 += u;
        s.y1 = fma(yv, u, s.y1);
        if (KERN == KR_EPANECHNIKOV) {
            const double u2 = u * u;
            s.u2 += u2;
            s.y2 = fma(yv, u2, s.y2);
        }
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
        // Shared-element moments.  Epanechnikov and uniform need only |d|^2
        // or nothing, so both sides share one set; triangular needs the sign
        // of (x_j - x_r), so it keeps one set per side.
        Shared sh0{0, 0, 0, 0, 0, 0}, sh1{0, 0, 0, 0, 0, 0};
        Shared &shR = sh0;
        Shared &shL = (KERN == KR_TRIANGULAR) ? sh1 : sh0;

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
                // Fast path (right): row 0 is the laggard; if its 4th element is
                // inside and no row has already counted any of the quad, every
                // row takes all four -> shared moments (7 FP64 per element for
                // G pairs).
                bool rfast = false;
                double u3 = 0.0;
                if (rgo) {
                    u3 = a[3].x - xr[0];
                    rfast = pR >= nx[G - 1] && inside<KERN>(u3, h);
                }
                if (rfast) {
#pragma unroll
                    for (int q = 0; q < 4; q++) sh_add<KERN>(shR, a[q].y, q == 3 ? u3 : a[q].x - xr[0]);
                    pR += 4 * G;
#pragma unroll
                    for (int r = 0; r < G; r++) nx[r] = pR;
                } else if (rgo) {
                    int ndone = 0;  // rows whose window ended: a prefix 0..ndone-1
#pragma unroll
                    for (int r = 0; r < G; r++) {
                        int cnt = 0;
#pragma unroll
                        for (int q = 0; q < 4; q++) {
                            const double d = a[q].x - xr[r];
                            const bool in = inside<KERN>(d, h);
                            cnt += in ? 1 : 0;
                            if (in && pR + q * G >= nx[r]) acc<KERN>(sR[r], a[q].y, d);
                        }
                        // first outside element of row r = pR + cnt*G, but only in
                        // the quad where row r's inside-prefix ends (cnt > 0);
                        // later quads of this bucket lie wholly outside row r.
                        if (cnt) nx[r] = max(nx[r], pR + cnt * G);
                        if (cnt < 4) ndone = r + 1;
                    }
                    // continue from the laggard among the rows still inside;
                    // jump over elements every active row has already counted
                    rgo = ndone < G;
                    int nxt = pR + 4 * G;
#pragma unroll
                    for (int r = 0; r < G; r++)
                        if (r == ndone) nxt = max(nxt, nx[r]);
                    pR = nxt;
                }
                // Fast path (left): row G-1 is the laggard.
                bool lfast = false;
                if (lgo) lfast = pL <= pv[0] && inside<KERN>(xr[G - 1] - c[3].x, h);
                if (lfast) {
#pragma unroll
                    for (int q = 0; q < 4; q++) sh_add<KERN>(shL, c[q].y, c[q].x - xr[0]);
                    pL -= 4 * G;
#pragma unroll
                    for (int r = 0; r < G; r++) pv[r] = pL;
                } else if (lgo) {
                    int nact = G;  // rows still inside: a prefix 0..nact-1
#pragma unroll
                    for (int r = G - 1; r >= 0; r--) {
                        int cnt = 0;
#pragma unroll
                        for (int q = 0; q < 4; q++) {
                            const double d = xr[r] - c[q].x;
                            const bool in = inside<KERN>(d, h);
                            cnt += in ? 1 : 0;
                            if (in && pL - q * G <= pv[r]) acc<KERN>(sL[r], c[q].y, d);
                        }
                        if (cnt) pv[r] = min(pv[r], pL - cnt * G);
                        if (cnt < 4) nact = r;
                    }
                    lgo = nact > 0;
                    int nxt = pL - 4 * G;
#pragma unroll
                    for (int r = 0; r < G; r++)
                        if (r == nact - 1) nxt = min(nxt, pv[r]);
                    pL = nxt;
                }
            }

            // ---- a4: reduce-scatter -> lane k owns row i0 + k
            int cRv[G], cLv[G];
            double syv[G], s1v[G], sy1v[G];
#pragma unroll
            for (int r = 0; r < G; r++) {
                cRv[r] = (nx[r] - first_n[r]) / G;
                cLv[r] = (first_p[r] - pv[r]) / G;
                syv[r] = sR[r].sy + sL[r].sy + shR.y0;
                s1v[r] = sR[r].s1 + sL[r].s1;
                sy1v[r] = sR[r].sy1 + sL[r].sy1;
                const double dl = xr[r] - xr[0];  // delta_r
                if (KERN == KR_EPANECHNIKOV) {
                    s1v[r] += fma(dl * dl, shR.c, fma(-2.0 * dl, shR.u1, shR.u2));
                    sy1v[r] += fma(dl * dl, shR.y0, fma(-2.0 * dl, shR.y1, shR.y2));
                } else if (KERN == KR_TRIANGULAR) {
                    syv[r] += shL.y0;
                    s1v[r] += fma(-dl, shR.c, shR.u1) + fma(dl, shL.c, -shL.u1);
                    sy1v[r] += fma(-dl, shR.y0, shR.y1) + fma(dl, shL.y0, -shL.y1);
                }
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
