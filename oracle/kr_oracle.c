/*
 * kr_oracle.c -- CPU ORACLE for the leave-one-out CV bandwidth grid search.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_rohlfsz17_b200/csrc); neither includes the other.
 *
 * What it computes (PAPER.md = Rohlfs & Zahran, IPDPSW 2017; citations are
 * P@<char offset> into the single-line PAPER.md):
 *
 *   Eq.(1) P@11484  CV(h) = n^-1 sum_i (Y_i - g_{-i}(X_i))^2 M(X_i)
 *   Eq.(2) P@11694  g_{-i}(X_i) = sum_{l!=i} Y_l K((X_i-X_l)/h) / sum_{l!=i} K((X_i-X_l)/h)
 *          P@11802  M(X_i) = 1 iff the denominator of (2) is non-zero
 *   Eq.(3) P@11971  K(u) = 0.75 (1-u^2) I{|u|<=1}           (Epanechnikov)
 *   fn.1   P@18521  "The same approach can be used for the Uniform and
 *                   Triangular kernels"  -> K(u)=1/2 I{|u|<=1},
 *                   K(u)=(1-|u|) I{|u|<1}  (reading Q13, textbook forms)
 *   P@10203         "straightforward to add additional ones" -> Gaussian
 *                   K(u) = exp(-u^2/2) (the 1/sqrt(2 pi) cancels in (2));
 *                   direct evaluator only (reading Q23).
 *
 * Two independent evaluators:
 *
 *   kro_cv_direct  -- the plain definition, Eq.(1)-(3) written out:
 *                     for every bandwidth, every row, every other row.
 *                     O(n^2 m).  No sort, no running sums.
 *   kro_cv_sorted  -- the paper's own algorithm (Program 3 "Sequential C",
 *                     P@27641, P@28414; §III P@13614-14984; §IV.B
 *                     P@20401-22459): per row, fill |X_i - X_l|, sort,
 *                     sweep the ascending grid carrying the running sums
 *                     forward ("copy our sums ... and begin to add",
 *                     P@21724), then divide by h^2, multiply by 0.75,
 *                     form (Y_i - g)^2 M.
 *
 * Readings of the paper used here:
 *   Q1  window membership is decided in IEEE binary64 on d = fabs(x_l - x_i):
 *       d <  h for Epanechnikov and triangular, d <= h for uniform.
 *   Q6  M_i = [number of in-window l != i >= 1] (integer test).
 *   Q7  rows with M_i = 0 contribute 0; CV divides by n (Eq.(1) literally).
 *   Q8  leave-one-out excludes the index i only (duplicates of X_i stay).
 *   Q11 best = smallest b with minimal CV; NaN is never minimal.
 *   Q12 arithmetic in long double (KRO_REAL), inputs are binary64.
 *   Q23 Gaussian: every l != i is in the window (full support), M_i = 1 for
 *       n >= 2; numerator and denominator of (2) are both multiplied by
 *       exp(dmin_i^2 / (2 h^2)), dmin_i = min_{l != i} |x_l - x_i| (an exact
 *       identity), so the nearest neighbour has weight 1 and no weight
 *       underflow can turn (2) into 0/0.
 *   Q14 the sorted sweep's decomposition h^2 c - sum d^2 cancels when all
 *       in-window points sit near the edge; if 0.75(c - sum d^2/h^2) <
 *       2^-30 * 0.75 c it recomputes numerator and denominator directly from
 *       K over the sorted prefix (the direct form has no cancellation).
 *
 * Determinism: row work is split in fixed chunks whose partial sums are
 * added in chunk order, so results do not depend on the thread count.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#ifndef KRO_REAL
#define KRO_REAL long double
#endif
typedef KRO_REAL real;

#define KRO_UNIFORM 0
#define KRO_EPANECHNIKOV 1
#define KRO_TRIANGULAR 2
#define KRO_GAUSSIAN 3

#define KRO_OK 0
#define KRO_EARG 1
#define KRO_EKERNEL 2
#define KRO_EGRID 3
#define KRO_ENONFINITE 4
#define KRO_EDEGENERATE 5
#define KRO_ENOMEM 6

#define KRO_MAX_M 65536
#define KRO_CHUNK 256

/* ------------------------------------------------------------------ */
/* validation: same contract as the C-ABI, own code   */
/* ------------------------------------------------------------------ */
static int kro_validate(const double *x, const double *y, int64_t n,
                        const double *h, int32_t m, int32_t kernel)
{
    if (!x || !y || !h) return KRO_EARG;
    if (n < 2 || n > 2147483647LL || m < 1 || m > KRO_MAX_M) return KRO_EARG;
    if (kernel != KRO_UNIFORM && kernel != KRO_EPANECHNIKOV && kernel != KRO_TRIANGULAR &&
        kernel != KRO_GAUSSIAN)
        return KRO_EKERNEL;
    for (int32_t b = 0; b < m; b++) {
        if (!isfinite(h[b]) || !(h[b] > 0.0)) return KRO_EGRID;
        if (b > 0 && h[b] < h[b - 1]) return KRO_EGRID;
    }
    for (int64_t i = 0; i < n; i++)
        if (!isfinite(x[i]) || !isfinite(y[i])) return KRO_ENONFINITE;
    return KRO_OK;
}

/* Q1: the window predicate, binary64 (Gaussian: full support, Q23). */
static int in_window(double d, double h, int32_t kernel)
{
    if (kernel == KRO_GAUSSIAN) return 1;
    return kernel == KRO_UNIFORM ? (d <= h) : (d < h);
}

/* Eq.(3) and footnote 1 (Q13), with u = d/h, |u| inside the window. */
static real kernel_K(double d, double h, int32_t kernel)
{
    real u = (real)d / (real)h;
    switch (kernel) {
    case KRO_EPANECHNIKOV: return (real)0.75 * ((real)1 - u * u);
    case KRO_TRIANGULAR:   return (real)1 - u;
    default:               return (real)0.5;
    }
}

/* Default grid, §IV P@16146-16375: max = range of X, min = range/k, evenly
 * spaced; written h_b = r * ((b+1)/m) (reading Q9). */
int kro_default_grid(const double *x, int64_t n, int32_t m, double *h_out)
{
    if (!x || !h_out || n < 2 || m < 1 || m > KRO_MAX_M) return KRO_EARG;
    double lo = x[0], hi = x[0];
    for (int64_t i = 0; i < n; i++) {
        if (!isfinite(x[i])) return KRO_ENONFINITE;
        if (x[i] < lo) lo = x[i];
        if (x[i] > hi) hi = x[i];
    }
    double r = hi - lo;
    if (!(r > 0.0)) return KRO_EDEGENERATE;
    for (int32_t b = 0; b < m; b++) h_out[b] = r * ((double)(b + 1) / (double)m);
    return KRO_OK;
}

/* Eq.(1) finalize + Q11 arg-min.  S[b] = sum_i M_i e_i^2 (long double). */
static void kro_finish(const real *S, int64_t n, int32_t m, double *cv_out, int32_t *best_out)
{
    int32_t best = -1;
    for (int32_t b = 0; b < m; b++) {
        double cv = (double)(S[b] / (real)n);
        if (cv_out) cv_out[b] = cv;
        if (!isnan(cv) && (best < 0 || cv < (double)(S[best] / (real)n))) best = b;
    }
    if (best_out) *best_out = best < 0 ? 0 : best;
}

/* ------------------------------------------------------------------ */
/* Evaluator 1: the plain definition, Eq.(1)-(3).                      */
/* rows: optional list of row indices (NULL = all rows 0..n-1).         */
/* S_out[m]   : sum over the listed rows of M_i (Y_i - g_{-i})^2        */
/* neff_out[m]: sum over the listed rows of M_i                         */
/* csum_out, sysum_out, sd2sum_out (nullable, [m]): sum over rows of    */
/*   |W_i|, sum_{l in W_i} Y_l, sum_{l in W_i} d_il^2  (pins P7, P8)    */
/* ------------------------------------------------------------------ */
static int direct_core(const double *x, const double *y, int64_t n,
                       const double *h, int32_t m, int32_t kernel,
                       const int64_t *rows, int64_t nrows,
                       real *S, int64_t *neff, int64_t *csum, real *sysum, real *sd2sum)
{
    int64_t R = rows ? nrows : n;
#pragma omp parallel for schedule(dynamic, 1)
    for (int32_t b = 0; b < m; b++) {
        real Sb = 0, sy_b = 0, sd2_b = 0;
        int64_t ne = 0, cs = 0;
        for (int64_t r = 0; r < R; r++) {
            int64_t i = rows ? rows[r] : r;
            real num = 0, den = 0;      /* Eq.(2) numerator, denominator */
            int64_t cnt = 0;
            real dmin2 = 0;             /* Gaussian scaling, Q23 */
            if (kernel == KRO_GAUSSIAN) {
                double dmin = INFINITY;
                for (int64_t l = 0; l < n; l++)
                    if (l != i && fabs(x[l] - x[i]) < dmin) dmin = fabs(x[l] - x[i]);
                dmin2 = (real)dmin * (real)dmin;
            }
            for (int64_t l = 0; l < n; l++) {
                if (l == i) continue;                       /* l != i */
                double d = fabs(x[l] - x[i]);
                if (!in_window(d, h[b], kernel)) continue;  /* I{|u| <= 1} */
                real w = kernel == KRO_GAUSSIAN
                             ? expl(-((real)d * (real)d - dmin2) / ((real)2 * (real)h[b] * (real)h[b]))
                             : kernel_K(d, h[b], kernel);
                num += (real)y[l] * w;
                den += w;
                cnt++;
                sy_b += (real)y[l];
                sd2_b += (real)d * (real)d;
            }
            cs += cnt;
            if (cnt == 0) continue;                         /* M(X_i) = 0 */
            real e = (real)y[i] - num / den;
            Sb += e * e;
            ne++;
        }
        S[b] = Sb;
        neff[b] = ne;
        if (csum) csum[b] = cs;
        if (sysum) sysum[b] = sy_b;
        if (sd2sum) sd2sum[b] = sd2_b;
    }
    return KRO_OK;
}

int kro_cv_direct(const double *x, const double *y, int64_t n,
                  const double *h, int32_t m, int32_t kernel,
                  const int64_t *rows, int64_t nrows,
                  double *S_out, int64_t *neff_out,
                  int64_t *csum_out, double *sysum_out, double *sd2sum_out,
                  double *cv_out, int32_t *best_out)
{
    int st = kro_validate(x, y, n, h, m, kernel);
    if (st) return st;
    if (rows && nrows < 0) return KRO_EARG;
    if (rows)
        for (int64_t r = 0; r < nrows; r++)
            if (rows[r] < 0 || rows[r] >= n) return KRO_EARG;
    real *S = (real *)calloc((size_t)m, sizeof(real));
    real *sy = (real *)calloc((size_t)m, sizeof(real));
    real *sd2 = (real *)calloc((size_t)m, sizeof(real));
    int64_t *ne = (int64_t *)calloc((size_t)m, sizeof(int64_t));
    if (!S || !sy || !sd2 || !ne) { free(S); free(sy); free(sd2); free(ne); return KRO_ENOMEM; }
    st = direct_core(x, y, n, h, m, kernel, rows, nrows, S, ne, csum_out, sy, sd2);
    if (!st) {
        for (int32_t b = 0; b < m; b++) {
            if (S_out) S_out[b] = (double)S[b];
            if (neff_out) neff_out[b] = ne[b];
            if (sysum_out) sysum_out[b] = (double)sy[b];
            if (sd2sum_out) sd2sum_out[b] = (double)sd2[b];
        }
        kro_finish(S, n, m, cv_out, best_out);
    }
    free(S); free(sy); free(sd2); free(ne);
    return st;
}

/* ------------------------------------------------------------------ */
/* Evaluator 2: the paper's sorting-based sweep (Program 3).           */
/* ------------------------------------------------------------------ */
typedef struct { double d; double y; int64_t l; } kro_pair;

static int cmp_pair(const void *a, const void *b)
{
    const kro_pair *p = (const kro_pair *)a, *q = (const kro_pair *)b;
    if (p->d < q->d) return -1;
    if (p->d > q->d) return 1;
    return (p->l > q->l) - (p->l < q->l);
}

/* One row i: fill, sort, sweep, residuals.  Adds into S[m], ne[m]. */
static void sorted_row(const double *x, const double *y, int64_t n,
                       const double *h, int32_t m, int32_t kernel, int64_t i,
                       kro_pair *buf, real *S, int64_t *ne)
{
    const real tau = (real)1 / (real)1073741824.0; /* 2^-30, Q14 */
    /* "Each thread j fills in n values of the abs(X_i - X_j) and Y_i" P@20401 */
    int64_t k = 0;
    for (int64_t l = 0; l < n; l++) {
        if (l == i) continue; /* "the final sums exclude ... the j-th observation" P@22353 */
        buf[k].d = fabs(x[l] - x[i]);
        buf[k].y = y[l];
        buf[k].l = l;
        k++;
    }
    /* "it sorts both of these matrices in order of abs(X_i - X_j)" P@20459 */
    qsort(buf, (size_t)k, sizeof(kro_pair), cmp_pair);

    /* "We begin with the smallest bandwidth" P@21154 -- running sums carried
     * from bandwidth to bandwidth. §III P@14010: sums of Y_l, Y_l d^2, d^2;
     * plus the count c (reading Q3). Triangular: Y_l d and d (reading Q13). */
    int64_t p = 0;
    real c = 0, sy = 0, s2 = 0, sy2 = 0;
    for (int32_t b = 0; b < m; b++) {
        double hb = h[b];
        while (p < k && in_window(buf[p].d, hb, kernel)) {
            real d = (real)buf[p].d, yl = (real)buf[p].y;
            c += 1;
            sy += yl;
            if (kernel == KRO_EPANECHNIKOV) { s2 += d * d; sy2 += yl * d * d; }
            else if (kernel == KRO_TRIANGULAR) { s2 += d; sy2 += yl * d; }
            p++;
        }
        if (p == 0) continue; /* M(X_i) = 0: no in-window neighbour (Q6, Q7) */
        real H = (real)hb, g;
        if (kernel == KRO_UNIFORM) {
            g = ((real)0.5 * sy) / ((real)0.5 * c);
        } else {
            /* "divided by the square of the bandwidths and multiplied by 0.75" P@22188 */
            real num, den;
            if (kernel == KRO_EPANECHNIKOV) {
                num = (real)0.75 * (sy - sy2 / (H * H));
                den = (real)0.75 * (c - s2 / (H * H));
                if (!(den >= tau * (real)0.75 * c)) goto direct;
            } else {
                num = sy - sy2 / H;
                den = c - s2 / H;
                if (!(den >= tau * c)) goto direct;
            }
            g = num / den;
            goto emit;
        direct: /* Q14: recompute from K over the in-window prefix [0, p) */
            num = 0; den = 0;
            for (int64_t q = 0; q < p; q++) {
                real w = kernel_K(buf[q].d, hb, kernel);
                num += (real)buf[q].y * w;
                den += w;
            }
            g = num / den;
        }
    emit:;
        real e = (real)y[i] - g;
        S[b] += e * e;
        ne[b] += 1;
    }
}

int kro_cv_sorted(const double *x, const double *y, int64_t n,
                  const double *h, int32_t m, int32_t kernel,
                  const int64_t *rows, int64_t nrows,
                  double *S_out, int64_t *neff_out,
                  double *cv_out, int32_t *best_out)
{
    int st = kro_validate(x, y, n, h, m, kernel);
    if (st) return st;
    if (kernel == KRO_GAUSSIAN) return KRO_EKERNEL; /* no finite window to sweep (Q23) */
    int64_t R = rows ? nrows : n;
    if (R < 0) return KRO_EARG;
    if (rows)
        for (int64_t r = 0; r < R; r++)
            if (rows[r] < 0 || rows[r] >= n) return KRO_EARG;
    int64_t nchunks = (R + KRO_CHUNK - 1) / KRO_CHUNK;
    real *Sc = (real *)calloc((size_t)(nchunks ? nchunks : 1) * (size_t)m, sizeof(real));
    int64_t *nc = (int64_t *)calloc((size_t)(nchunks ? nchunks : 1) * (size_t)m, sizeof(int64_t));
    if (!Sc || !nc) { free(Sc); free(nc); return KRO_ENOMEM; }
    int oom = 0;
#pragma omp parallel
    {
        kro_pair *buf = (kro_pair *)malloc((size_t)n * sizeof(kro_pair));
        if (!buf) {
#pragma omp atomic write
            oom = 1;
        }
#pragma omp for schedule(dynamic, 1)
        for (int64_t ch = 0; ch < nchunks; ch++) {
            if (!buf) continue;
            int64_t r0 = ch * KRO_CHUNK, r1 = r0 + KRO_CHUNK < R ? r0 + KRO_CHUNK : R;
            for (int64_t r = r0; r < r1; r++) {
                int64_t i = rows ? rows[r] : r;
                sorted_row(x, y, n, h, m, kernel, i, buf, Sc + ch * m, nc + ch * m);
            }
        }
        free(buf);
    }
    if (oom) { free(Sc); free(nc); return KRO_ENOMEM; }
    /* "a summation reduction is performed k times, once for each bandwidth" P@23970;
     * chunk partials added in chunk order (deterministic). */
    real *S = (real *)calloc((size_t)m, sizeof(real));
    if (!S) { free(Sc); free(nc); return KRO_ENOMEM; }
    for (int32_t b = 0; b < m; b++) {
        real s = 0;
        int64_t ne = 0;
        for (int64_t ch = 0; ch < nchunks; ch++) { s += Sc[ch * m + b]; ne += nc[ch * m + b]; }
        S[b] = s;
        if (S_out) S_out[b] = (double)s;
        if (neff_out) neff_out[b] = ne;
    }
    kro_finish(S, n, m, cv_out, best_out);
    free(S); free(Sc); free(nc);
    return KRO_OK;
}

/* Public finalize for summed shard partials (mirrors the ABI's kr_finalize,
 * own code): CV[b] = S[b]/n, best per Q11. */
int kro_finalize(const double *S, int64_t n, int32_t m, double *cv_out, int32_t *best_out)
{
    if (!S || n < 1 || m < 1) return KRO_EARG;
    real *T = (real *)malloc((size_t)m * sizeof(real));
    if (!T) return KRO_ENOMEM;
    for (int32_t b = 0; b < m; b++) T[b] = (real)S[b];
    kro_finish(T, n, m, cv_out, best_out);
    free(T);
    return KRO_OK;
}

int kro_real_bits(void) { return (int)(sizeof(real) * 8); }

int kro_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ------------------------------------------------------------------ */
/* KDE least-squares cross-validation (PAPER.md P@10382-10640: "the     */
/* methods developed here for least-squares cross-validation can be     */
/* applied to ... optimal bandwidth selection for kernel density        */
/* estimation"; reading Q24).                   */
/*                                                                      */
/*   f_h(x)        = (1/(n h)) sum_j K((x - x_j)/h)                     */
/*   f_{h,-i}(x_i) = (1/((n-1) h)) sum_{j!=i} K((x_i - x_j)/h)          */
/*   LSCV(h)       = int f_h^2 - (2/n) sum_i f_{h,-i}(x_i)               */
/*   int f_h^2     = (1/(n^2 h)) sum_i sum_j Kbar((x_i - x_j)/h),        */
/*   Kbar = K * K (self-convolution), written out below.                */
/* Kernels normalised to integrate to 1 (Q24): uniform 1/2 I{|u|<=1},   */
/* Epanechnikov 3/4 (1-u^2) I{|u|<=1}, triangular (1-|u|) I{|u|<1}.     */
/* Window membership as Q1: K's window d <= h (uniform) / d < h, Kbar's */
/* d < 2h (Kbar vanishes continuously at |u| = 2 for all three).        */
/* The plain definition, O(n^2 m); per row i: A_i = sum_{j!=i} Kbar,    */
/* B_i = sum_{j!=i} K; LSCV = (n Kbar(0) + sum A)/(n^2 h)               */
/*                           - 2 sum B / (n (n-1) h).                   */
/* ------------------------------------------------------------------ */
static real kde_kbar(real v, int32_t kernel) /* v = |u| in [0, 2) */
{
    switch (kernel) {
    case KRO_EPANECHNIKOV: /* (3/160) (2-v)^3 (v^2 + 6 v + 4) */
        return (real)3 / (real)160 * (2 - v) * (2 - v) * (2 - v) * (v * v + 6 * v + 4);
    case KRO_TRIANGULAR:   /* cubic B-spline */
        if (v < 1) return (real)2 / (real)3 - v * v + v * v * v / 2;
        return (2 - v) * (2 - v) * (2 - v) / 6;
    default:               /* uniform: triangle */
        return (2 - v) / 4;
    }
}

static real kde_k(real v, int32_t kernel) /* v = |u| inside K's window */
{
    switch (kernel) {
    case KRO_EPANECHNIKOV: return (real)0.75 * (1 - v * v);
    case KRO_TRIANGULAR:   return 1 - v;
    default:               return (real)0.5;
    }
}

int kro_kde_lscv(const double *x, int64_t n, const double *h, int32_t m, int32_t kernel,
                 const int64_t *rows, int64_t nrows, double *A_out, double *B_out,
                 double *lscv_out, int32_t *best_out)
{
    if (!x || !h || n < 2 || m < 1 || m > KRO_MAX_M) return KRO_EARG;
    if (kernel != KRO_UNIFORM && kernel != KRO_EPANECHNIKOV && kernel != KRO_TRIANGULAR) return KRO_EKERNEL;
    for (int32_t b = 0; b < m; b++) {
        if (!isfinite(h[b]) || !(h[b] > 0.0)) return KRO_EGRID;
        if (b > 0 && h[b] < h[b - 1]) return KRO_EGRID;
    }
    for (int64_t i = 0; i < n; i++)
        if (!isfinite(x[i])) return KRO_ENONFINITE;
    int64_t R = rows ? nrows : n;
    if (R < 0) return KRO_EARG;
    real *A = (real *)calloc((size_t)m, sizeof(real));
    real *B = (real *)calloc((size_t)m, sizeof(real));
    if (!A || !B) { free(A); free(B); return KRO_ENOMEM; }
#pragma omp parallel for schedule(dynamic, 1)
    for (int32_t b = 0; b < m; b++) {
        const double hb = h[b], h2 = 2.0 * hb; /* 2h exact in binary64 */
        real Ab = 0, Bb = 0;
        for (int64_t r = 0; r < R; r++) {
            int64_t i = rows ? rows[r] : r;
            for (int64_t l = 0; l < n; l++) {
                if (l == i) continue;
                double d = fabs(x[l] - x[i]);
                real v = (real)d / (real)hb;
                if (d < h2) Ab += kde_kbar(v, kernel);
                if (in_window(d, hb, kernel)) Bb += kde_k(v, kernel);
            }
        }
        A[b] = Ab;
        B[b] = Bb;
    }
    int32_t best = -1;
    real bestv = 0;
    for (int32_t b = 0; b < m; b++) {
        if (A_out) A_out[b] = (double)A[b];
        if (B_out) B_out[b] = (double)B[b];
        if (!rows) {
            real nn = (real)n, hb = (real)h[b];
            real v = (nn * kde_kbar(0, kernel) + A[b]) / (nn * nn * hb) - 2 * B[b] / (nn * (nn - 1) * hb);
            if (lscv_out) lscv_out[b] = (double)v;
            if (!isnan((double)v) && (best < 0 || (double)v < (double)bestv)) { best = b; bestv = v; }
        }
    }
    if (best_out) *best_out = best < 0 ? 0 : best;
    free(A); free(B);
    return KRO_OK;
}

/* ------------------------------------------------------------------ */
/* Local-linear leave-one-out CV (PAPER.md      */
/* §IV P@15728-15905: "The Nadaraya-Watson [19], [27] local constant    */
/* estimator is used rather than a local linear regression" -- the      */
/* local-linear estimator is the named alternative; reading Q25).       */
/*                                                                      */
/* For row i and bandwidth h the LOO local-linear estimate is the       */
/* intercept a of the kernel-weighted least-squares line                */
/*   min_{a,beta} sum_{l != i, l in W_i} w_il (Y_l - a - beta d_il)^2,  */
/*   d_il = X_l - X_i (binary64), w_il = K(|d_il|/h) (Eq.(3), Q13),     */
/* over the same window W_i as Eq.(2) (reading Q1).  The 2x2 normal     */
/* equations are non-singular iff W_i holds at least two distinct X     */
/* values (all weights are > 0 inside the window), so                   */
/*   M_i = [W_i holds >= 2 distinct X]  (an integer test, as Q6),       */
/* rows with M_i = 0 contribute 0 and CV divides by n (as Q7).          */
/* The intercept is written in the centred (two-pass) form of the       */
/* weighted least-squares solution, algebraically identical to          */
/* (S2 T0 - S1 T1) / (S0 S2 - S1^2) with S_k = sum w d^k,               */
/* T_k = sum w Y d^k:                                                   */
/*   dbar = sum w d / sum w,  ybar = sum w Y / sum w,                   */
/*   beta = sum w (d - dbar)(Y - ybar) / sum w (d - dbar)^2,            */
/*   a    = ybar - beta dbar.                                           */
/* The plain definition: O(n) per (row, bandwidth), no sort.            */
/* ------------------------------------------------------------------ */
static int ll_row(const double *x, const double *y, int64_t n, double hb, int32_t kernel, int64_t i, real *e2)
{
    real s0 = 0, sd = 0, sy = 0;
    int64_t first = -1, distinct = 0;
    for (int64_t l = 0; l < n; l++) {
        if (l == i) continue;
        double d = x[l] - x[i];
        if (!in_window(fabs(d), hb, kernel)) continue;
        real w = kernel_K(fabs(d), hb, kernel);
        s0 += w;
        sd += w * (real)d;
        sy += w * (real)y[l];
        if (first < 0) first = l;
        else if (x[l] != x[first]) distinct = 1;
    }
    if (!distinct) return 0; /* M_i = 0 */
    real dbar = sd / s0, ybar = sy / s0, sdd = 0, sdy = 0;
    for (int64_t l = 0; l < n; l++) {
        if (l == i) continue;
        double d = x[l] - x[i];
        if (!in_window(fabs(d), hb, kernel)) continue;
        real w = kernel_K(fabs(d), hb, kernel);
        real dc = (real)d - dbar;
        sdd += w * dc * dc;
        sdy += w * dc * ((real)y[l] - ybar);
    }
    real a = ybar - (sdy / sdd) * dbar;
    real e = (real)y[i] - a;
    *e2 = e * e;
    return 1;
}

int kro_ll_cv(const double *x, const double *y, int64_t n, const double *h, int32_t m, int32_t kernel,
              const int64_t *rows, int64_t nrows, double *S_out, int64_t *neff_out, double *cv_out,
              int32_t *best_out)
{
    int st = kro_validate(x, y, n, h, m, kernel);
    if (st) return st;
    if (kernel == KRO_GAUSSIAN) return KRO_EKERNEL;
    int64_t R = rows ? nrows : n;
    if (R < 0) return KRO_EARG;
    if (rows)
        for (int64_t r = 0; r < R; r++)
            if (rows[r] < 0 || rows[r] >= n) return KRO_EARG;
    real *S = (real *)calloc((size_t)m, sizeof(real));
    int64_t *ne = (int64_t *)calloc((size_t)m, sizeof(int64_t));
    if (!S || !ne) { free(S); free(ne); return KRO_ENOMEM; }
#pragma omp parallel for schedule(dynamic, 1)
    for (int32_t b = 0; b < m; b++) {
        real Sb = 0;
        int64_t nb = 0;
        for (int64_t r = 0; r < R; r++) {
            int64_t i = rows ? rows[r] : r;
            real e2 = 0;
            if (ll_row(x, y, n, h[b], kernel, i, &e2)) { Sb += e2; nb++; }
        }
        S[b] = Sb;
        ne[b] = nb;
    }
    for (int32_t b = 0; b < m; b++) {
        if (S_out) S_out[b] = (double)S[b];
        if (neff_out) neff_out[b] = ne[b];
    }
    kro_finish(S, n, m, cv_out, best_out);
    free(S); free(ne);
    return KRO_OK;
}

/* ------------------------------------------------------------------ */
/* Leave-one-out (delete-one jackknife) confidence intervals at a given */
/* bandwidth -- the CV-optimal one in use (§II P@10560-10640:  */
/* "the estimation of leave-one-out cross-validated confidence          */
/* intervals for kernel density estimates and kernel regressions";      */
/* SURVEY.md §8(f) rank 3; reading Q26).                     */
/*                                                                      */
/* Kernel regression (Nadaraya-Watson, Eq.(2) with the point itself):   */
/*   W+_i = { j : d_ij in the window (Q1) }  (i itself included, d = 0) */
/*   w_ij = K(d_ij / h) (Eq.(3), Q13), D_i = sum w_ij,                  */
/*   N_i = sum w_ij Y_j, g_i = N_i / D_i                                */
/*   delete-one estimates g_i^(-j) = (N_i - w_ij Y_j) / (D_i - w_ij)    */
/*   (= g_i for j outside W+_i), jackknife variance                     */
/*   V_i = (n-1)/n sum_j (g_i^(-j) - mean_j g_i^(-j))^2                 */
/* written with Delta_j = g_i^(-j) - g_i = -w_ij (Y_j - g_i)/(D_i-w_ij) */
/* (zero outside W+_i) as                                               */
/*   V_i = (n-1)/n [ sum Delta_j^2 - (sum Delta_j)^2 / n ].             */
/* A point whose window holds only itself has no delete-one estimate at */
/* j = i: its se is NaN (no interval).  Output in the caller's order.   */
/*                                                                      */
/* Kernel density (Q24's normalised kernels):                           */
/*   K_ij = K(d_ij / h) / h on K's window, f_i = (1/n) sum_j K_ij       */
/*   delete-one f_i^(-j) = (n f_i - K_ij)/(n-1); its jackknife variance */
/*   reduces to the sample variance of the K_ij over j = 0..n-1:        */
/*   V_i = sum_j (K_ij - f_i)^2 / (n (n-1))                             */
/*       = [ sum_{W+} (K_ij - f_i)^2 + (n - |W+_i|) f_i^2 ] / (n(n-1)). */
/* The interval is est_i -+ z se_i, se_i = sqrt(V_i) (z from the        */
/* caller's level).  Both: the plain definitions, O(n) per point.       */
/* ------------------------------------------------------------------ */
int kro_nw_jackknife(const double *x, const double *y, int64_t n, double h, int32_t kernel,
                     double *est_out, double *se_out, int64_t *nwin_out)
{
    if (!x || !y || !est_out || !se_out || n < 2) return KRO_EARG;
    if (kernel != KRO_UNIFORM && kernel != KRO_EPANECHNIKOV && kernel != KRO_TRIANGULAR) return KRO_EKERNEL;
    if (!isfinite(h) || !(h > 0.0)) return KRO_EGRID;
    for (int64_t i = 0; i < n; i++)
        if (!isfinite(x[i]) || !isfinite(y[i])) return KRO_ENONFINITE;
    const real nn = (real)n;
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t i = 0; i < n; i++) {
        real D = 0, N = 0;
        int64_t c = 0;
        for (int64_t j = 0; j < n; j++) {
            double d = fabs(x[j] - x[i]);
            if (!in_window(d, h, kernel)) continue;
            real w = kernel_K(d, h, kernel);
            D += w;
            N += w * (real)y[j];
            c++;
        }
        real g = N / D;
        real s1 = 0, s2 = 0;
        int ok = 1;
        for (int64_t j = 0; j < n; j++) {
            double d = fabs(x[j] - x[i]);
            if (!in_window(d, h, kernel)) continue;
            real w = kernel_K(d, h, kernel);
            real rest = D - w;
            if (!(rest > 0)) { ok = 0; break; }
            real delta = -w * ((real)y[j] - g) / rest;
            s1 += delta;
            s2 += delta * delta;
        }
        est_out[i] = (double)g;
        se_out[i] = ok ? (double)sqrtl((nn - 1) / nn * (s2 - s1 * s1 / nn)) : NAN;
        if (nwin_out) nwin_out[i] = c;
    }
    return KRO_OK;
}

int kro_kde_jackknife(const double *x, int64_t n, double h, int32_t kernel, double *est_out, double *se_out)
{
    if (!x || !est_out || !se_out || n < 2) return KRO_EARG;
    if (kernel != KRO_UNIFORM && kernel != KRO_EPANECHNIKOV && kernel != KRO_TRIANGULAR) return KRO_EKERNEL;
    if (!isfinite(h) || !(h > 0.0)) return KRO_EGRID;
    for (int64_t i = 0; i < n; i++)
        if (!isfinite(x[i])) return KRO_ENONFINITE;
    const real nn = (real)n, hh = (real)h;
#pragma omp parallel for schedule(dynamic, 64)
    for (int64_t i = 0; i < n; i++) {
        real S = 0;
        int64_t c = 0;
        for (int64_t j = 0; j < n; j++) {
            double d = fabs(x[j] - x[i]);
            if (!in_window(d, h, kernel)) continue;
            S += kde_k((real)d / hh, kernel) / hh;
            c++;
        }
        real f = S / nn;
        real q = 0;
        for (int64_t j = 0; j < n; j++) {
            double d = fabs(x[j] - x[i]);
            if (!in_window(d, h, kernel)) continue;
            real t = kde_k((real)d / hh, kernel) / hh - f;
            q += t * t;
        }
        q += (nn - (real)c) * f * f;
        est_out[i] = (double)f;
        se_out[i] = (double)sqrtl(q / (nn * (nn - 1)));
    }
    return KRO_OK;
}
