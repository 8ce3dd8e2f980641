/* A plain-C consumer of the C-ABI (include/krcv.h, libkrcv.so): no Python,
 * no PyTorch.  Builds the paper's synthetic design (PAPER.md P@16457:
 * X ~ U(0,1), Y = 0.5 X + 10 X^2 + U(0, 0.5)), the default grid (§IV
 * P@16146) and runs the LOO-CV grid search on the current GPU.
 *
 *   gcc -O2 -I include examples/krcv_example.c \
 *       -L paper_conf_ipps_rohlfsz17_b200 -lkrcv \
 *       -Wl,-rpath,$PWD/paper_conf_ipps_rohlfsz17_b200 -o krcv_example
 *   ./krcv_example [n] [m] [--dump] (--host-only: ABI checks without a GPU)
 *
 * --dump prints the whole CV curve and n_eff (kr_cv_grid_ex) and the
 * leave-one-out confidence intervals at the optimum (kr_cv_ci) of every
 * observation, one value per line in %.17g, for tests/test_c_consumer.py.
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "krcv.h"

static uint64_t s = 0x9E3779B97F4A7C15ull;
static double urand(void)
{
    s ^= s << 13;
    s ^= s >> 7;
    s ^= s << 17;
    return (double)(s >> 11) * 0x1p-53;
}

int main(int argc, char **argv)
{
    const int host_only = argc > 1 && strcmp(argv[1], "--host-only") == 0;
    const int64_t n = (!host_only && argc > 1) ? atoll(argv[1]) : 20000;
    const int32_t m = (!host_only && argc > 2) ? atoi(argv[2]) : 200;
    double *x = malloc(sizeof(double) * n), *y = malloc(sizeof(double) * n);
    double *h = malloc(sizeof(double) * m), *cv = malloc(sizeof(double) * m);
    if (!x || !y || !h || !cv) return 2;
    for (int64_t i = 0; i < n; i++) {
        x[i] = urand();
        y[i] = 0.5 * x[i] + 10.0 * x[i] * x[i] + 0.5 * urand();
    }
    printf("%s\n", kr_version());
    int st = kr_default_grid(x, n, m, h);
    if (st) { fprintf(stderr, "kr_default_grid: %s\n", kr_strerror(st)); return 1; }
    if (kr_validate_grid(h, m) != KR_OK) return 1;
    double bad[2] = {0.2, 0.1};
    if (kr_validate_grid(bad, 2) != KR_EGRID) return 1; /* decreasing grid rejected */
    int32_t best = -1;
    if (kr_cv_grid(x, y, 1, h, m, KR_EPANECHNIKOV, cv, &best) != KR_EARG) return 1; /* n < 2 */
    if (host_only) {
        printf("host-only ABI checks: ok (h[0] = %.9g, h[m-1] = %.9g)\n", h[0], h[m - 1]);
        return 0;
    }
    st = kr_cv_grid(x, y, n, h, m, KR_EPANECHNIKOV, cv, &best);
    if (st) { fprintf(stderr, "kr_cv_grid: %s (%s)\n", kr_strerror(st), kr_last_cuda_error()); return 1; }
    printf("n = %lld, m = %d: best b = %d, h = %.9g, CV = %.12g\n", (long long)n, m, best, h[best], cv[best]);
    if (argc > 3 && strcmp(argv[3], "--dump") == 0) {
        int64_t *neff = malloc(sizeof(int64_t) * m);
        double *est = malloc(sizeof(double) * n), *se = malloc(sizeof(double) * n);
        int32_t best2 = -1, best3 = -1;
        if (!neff || !est || !se) return 2;
        st = kr_cv_grid_ex(x, y, n, h, m, KR_EPANECHNIKOV, cv, neff, &best2);
        if (st || best2 != best) { fprintf(stderr, "kr_cv_grid_ex: %s\n", kr_strerror(st)); return 1; }
        for (int32_t b = 0; b < m; b++) printf("curve %d %.17g %lld\n", b, cv[b], (long long)neff[b]);
        st = kr_cv_ci(x, y, n, h, m, KR_EPANECHNIKOV, cv, est, se, &best3);
        if (st || best3 != best) { fprintf(stderr, "kr_cv_ci: %s\n", kr_strerror(st)); return 1; }
        for (int64_t i = 0; i < n; i++) printf("ci %lld %.17g %.17g\n", (long long)i, est[i], se[i]);
        free(neff); free(est); free(se);
    }
    kr_release();
    free(x); free(y); free(h); free(cv);
    return 0;
}
