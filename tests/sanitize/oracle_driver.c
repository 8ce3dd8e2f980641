/* T7: drive every oracle entry point on small inputs under
 * AddressSanitizer + UndefinedBehaviorSanitizer (tests/test_sanitizers_cpu.py
 * compiles oracle/kr_oracle.c together with this file).  Inputs: a random
 * design with duplicate x and points exactly at a bandwidth, n = 2, row
 * subsets, and the error paths (NaN, bad grid, unknown kernel, n < 2).
 * Test infrastructure only; exits non-zero on an unexpected status. */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

int kro_default_grid(const double *x, int64_t n, int32_t m, double *h_out);
int kro_cv_direct(const double *x, const double *y, int64_t n, const double *h, int32_t m, int32_t kernel,
                  const int64_t *rows, int64_t nrows, double *S_out, int64_t *neff_out, int64_t *csum_out,
                  double *sysum_out, double *sd2sum_out, double *cv_out, int32_t *best_out);
int kro_cv_sorted(const double *x, const double *y, int64_t n, const double *h, int32_t m, int32_t kernel,
                  const int64_t *rows, int64_t nrows, double *S_out, int64_t *neff_out, double *cv_out,
                  int32_t *best_out);
int kro_finalize(const double *S, int64_t n, int32_t m, double *cv_out, int32_t *best_out);
int kro_kde_lscv(const double *x, int64_t n, const double *h, int32_t m, int32_t kernel, const int64_t *rows,
                 int64_t nrows, double *A_out, double *B_out, double *lscv_out, int32_t *best_out);
int kro_ll_cv(const double *x, const double *y, int64_t n, const double *h, int32_t m, int32_t kernel,
              const int64_t *rows, int64_t nrows, double *S_out, int64_t *neff_out, double *cv_out,
              int32_t *best_out);

static int fails = 0;
#define EXPECT(cond, what)                                   \
    do {                                                     \
        if (!(cond)) {                                       \
            fprintf(stderr, "FAIL %s (line %d)\n", what, __LINE__); \
            fails++;                                         \
        }                                                    \
    } while (0)

static uint64_t rng = 88172645463325252ull;
static double urand(void)
{
    rng ^= rng << 13;
    rng ^= rng >> 7;
    rng ^= rng << 17;
    return (double)(rng >> 11) * 0x1p-53;
}

int main(void)
{
    enum { N = 300, M = 12 };
    double x[N], y[N], h[M], cv[M], S[M], A[M], B[M], sy[M], sd2[M];
    int64_t ne[M], cs[M], rows[17];
    int32_t best = -1;
    for (int i = 0; i < N; i++) {
        x[i] = floor(urand() * 64.0) / 16.0; /* dyadic: duplicates and exact distances */
        y[i] = urand() * 4.0 - 2.0;
    }
    EXPECT(kro_default_grid(x, N, M, h) == 0, "default grid");
    h[3] = 0.25; /* a pair distance exactly */
    h[4] = 0.25; /* duplicated grid point */
    for (int b = 1; b < M; b++)
        if (h[b] < h[b - 1]) h[b] = h[b - 1];
    for (int i = 0; i < 17; i++) rows[i] = (i * 37) % N;
    for (int k = 0; k < 4; k++) {
        EXPECT(kro_cv_direct(x, y, N, h, M, k, NULL, 0, S, ne, cs, sy, sd2, cv, &best) == 0, "direct");
        EXPECT(best >= 0 && best < M, "direct best");
        EXPECT(kro_cv_direct(x, y, N, h, M, k, rows, 17, S, ne, NULL, NULL, NULL, cv, &best) == 0, "direct rows");
        EXPECT(kro_finalize(S, N, M, cv, &best) == 0, "finalize");
        if (k < 3) {
            EXPECT(kro_cv_sorted(x, y, N, h, M, k, NULL, 0, S, ne, cv, &best) == 0, "sorted");
            EXPECT(kro_cv_sorted(x, y, N, h, M, k, rows, 17, S, ne, cv, &best) == 0, "sorted rows");
            EXPECT(kro_kde_lscv(x, N, h, M, k, NULL, 0, A, B, cv, &best) == 0, "kde");
            EXPECT(kro_kde_lscv(x, N, h, M, k, rows, 17, A, B, cv, &best) == 0, "kde rows");
            EXPECT(kro_ll_cv(x, y, N, h, M, k, NULL, 0, S, ne, cv, &best) == 0, "ll");
            EXPECT(kro_ll_cv(x, y, N, h, M, k, rows, 17, S, ne, cv, &best) == 0, "ll rows");
        }
        /* n = 2 */
        EXPECT(kro_cv_direct(x, y, 2, h, M, k, NULL, 0, S, ne, NULL, NULL, NULL, cv, &best) == 0, "direct n=2");
    }
    /* error paths: every one must return a non-zero status, touching nothing */
    double xb[N];
    for (int i = 0; i < N; i++) xb[i] = x[i];
    xb[7] = NAN;
    EXPECT(kro_cv_direct(xb, y, N, h, M, 1, NULL, 0, S, ne, NULL, NULL, NULL, cv, &best) != 0, "nan x");
    EXPECT(kro_cv_sorted(xb, y, N, h, M, 1, NULL, 0, S, ne, cv, &best) != 0, "nan x sorted");
    double hb[M];
    for (int b = 0; b < M; b++) hb[b] = h[M - 1 - b]; /* decreasing */
    EXPECT(kro_cv_sorted(x, y, N, hb, M, 1, NULL, 0, S, ne, cv, &best) != 0, "bad grid");
    EXPECT(kro_cv_direct(x, y, N, h, M, 9, NULL, 0, S, ne, NULL, NULL, NULL, cv, &best) != 0, "bad kernel");
    EXPECT(kro_cv_direct(x, y, 1, h, M, 1, NULL, 0, S, ne, NULL, NULL, NULL, cv, &best) != 0, "n<2");
    EXPECT(kro_ll_cv(x, y, N, h, M, 3, NULL, 0, S, ne, cv, &best) != 0, "ll gaussian");
    if (fails) return 1;
    printf("oracle sanitizer driver: ok\n");
    return 0;
}
