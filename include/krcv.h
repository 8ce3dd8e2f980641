/*
 * krcv.h -- C-ABI of the B200-native leave-one-out cross-validation
 * bandwidth grid search for univariate Nadaraya-Watson regression
 * (Rohlfs & Zahran, "Optimal Bandwidth Selection for Kernel Regression Using
 * a Fast Grid Search and a GPU", IPDPSW 2017).
 *
 * Citations are P@<char offset> into the single-line reference PAPER.md
 * (SURVEY.md §0).
 *
 * What is computed (§III):
 *   Eq.(1) P@11484  CV(h) = n^-1 sum_i (Y_i - g_{-i}(X_i))^2 M(X_i)
 *   Eq.(2) P@11694  g_{-i}(X_i) = sum_{l!=i} Y_l K((X_i-X_l)/h) / sum_{l!=i} K((X_i-X_l)/h)
 *          P@11802  M(X_i) = 1 iff the denominator of (2) is non-zero
 *   Eq.(3) P@11971  Epanechnikov K(u) = 0.75 (1-u^2) I{|u|<=1}
 *   fn.1   P@18521  uniform K = 1/2 I{|u|<=1}, triangular K = (1-|u|) I{|u|<1}
 * for every bandwidth h_b of a non-decreasing grid, then the arg-min
 * (§IV.B P@23454-26269; footnote 2 P@25449: return the index).
 *
 * Conventions:
 *   - Window membership is decided in IEEE binary64 on d = |x_l - x_i|:
 *     d < h for Epanechnikov / triangular, d <= h for uniform (Q1).
 *   - M_i = 1 iff at least one l != i is in the window (Q6).  Rows with
 *     M_i = 0 contribute 0 and CV divides by n (Eq.(1) literally, Q7).
 *   - Leave-one-out excludes index i only; duplicates of x_i stay (Q8).
 *   - best = smallest b whose CV equals the minimum; NaN is never minimal (Q11).
 *   - Arithmetic is fp64 (the paper's fp32, P@19633, misses 1e-6 parity).
 *   - Indices are 0-based.  The grid must be finite, > 0, non-decreasing;
 *     duplicates are allowed (equal CV, lower index wins).  No 2,048 cap
 *     (the paper's cap is a constant-memory artefact, P@20037).
 *
 * Ownership: the caller owns every buffer.  The library keeps no pointer to
 * caller memory after a call returns (async calls: until the enqueued stream
 * work completes).  Outputs are written only when a call returns KR_OK
 * (async calls: see the status slots of the partial vector).
 *
 * Threading: every entry point is re-entrant.  kr_cv_grid serialises on a
 * per-device context (lazily created workspace + stream) guarded by a mutex.
 */
#ifndef KRCV_H
#define KRCV_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Kernel functions K (Eq.(3), footnote 1 P@18521). */
enum {
    KR_UNIFORM = 0,
    KR_EPANECHNIKOV = 1,
    KR_TRIANGULAR = 2,
    KR_GAUSSIAN = 3  /* K(u) = exp(-u^2/2), P@10203 "additional [kernels]"; reading Q23:
                        full support, M_i = 1, weights rescaled by the nearest
                        neighbour's (exact for Eq.(2)); dense path only */
};

/* Status codes returned by every int-valued entry point. */
enum {
    KR_OK = 0,
    KR_EARG = 1,        /* null pointer, n < 2, n > INT32_MAX, m < 1, m > KR_MAX_M,
                           bad shard/nshards, workspace too small */
    KR_EKERNEL = 2,     /* unknown kernel id */
    KR_EGRID = 3,       /* h non-finite, h <= 0, or decreasing */
    KR_ENONFINITE = 4,  /* NaN / Inf in x or y */
    KR_EDEGENERATE = 5, /* default grid requested with max(x) == min(x) */
    KR_ENOMEM = 6,      /* device or host allocation failed */
    KR_ECUDA = 7        /* any other CUDA runtime error (see kr_last_cuda_error) */
};

#define KR_MAX_M 65536

/* Algorithms (both compute the same CV curve):
 *   KR_ALGO_SWEEP  the paper's per-row running sums (§III P@14010-14984,
 *                  §IV.B P@21724-22104): every row visits its neighbours in
 *                  distance order and adds them one by one as h grows --
 *                  O(n^2) pair steps + O(n m) emits;
 *   KR_ALGO_PREFIX window-prefix: the same running sums reached by exact
 *                  boundary search on the sorted x and differences of
 *                  double-double prefix moments --
 *                  O(n m log) work, no per-pair step;
 *   KR_ALGO_AUTO   the library's choice (currently KR_ALGO_PREFIX; the
 *                  environment variable KRCV_ALGO=sweep|prefix overrides). */
enum {
    KR_ALGO_AUTO = 0,
    KR_ALGO_SWEEP = 1,
    KR_ALGO_PREFIX = 2,
    KR_ALGO_DENSE = 3,  /* tiled all-pairs x all-bandwidths, the only path for
                           KR_GAUSSIAN (AUTO picks it); KR_EARG with the
                           compact kernels, and SWEEP / PREFIX / HIST give
                           KR_EARG with KR_GAUSSIAN */
    KR_ALGO_HIST = 4    /* bucket-by-bandwidth shared-memory histogram + warp
                           scan (north_star's named alternative to a per-row
                           sort; SURVEY.md §7.1 "H", an ablation -- never
                           chosen by AUTO): O(n^2) bucketed pairs with
                           shared-memory atomics; sums agree with the other
                           paths to rounding, not bitwise (atomic order).
                           Grids larger than one shared-memory histogram
                           (m > ~4,800) run in slices of ~2,600 bandwidths,
                           one O(n^2) pass each */
};

/* Length of the partial vector of the device path: [ S[0..m) | neff[0..m) |
 * n_bad_grid | n_nonfinite ].  S[b] = sum over the shard's rows of
 * M_i (y_i - g_{-i}(h_b))^2, neff[b] = sum of M_i (exact in fp64), and two
 * status counters.  All entries add under an all-reduce(SUM) across shards. */
#define KR_PARTIAL_LEN(m) (2 * (int64_t)(m) + 2)

/*
 * kr_cv_grid -- the whole grid search on the current CUDA device, host
 * pointers, synchronous.  (BASELINE.json north_star signature.)
 *   x, y     [n] fp64 host arrays (any order; any pageable or pinned memory)
 *   h_grid   [m] fp64 host, non-decreasing, finite, > 0
 *   kernel   KR_UNIFORM | KR_EPANECHNIKOV | KR_TRIANGULAR
 *   cv_out   [m] host: CV(h_b) per Eq.(1) (already divided by n)
 *   best_out host: smallest arg-min index
 * Errors: KR_EARG, KR_EKERNEL, KR_EGRID (arguments and grid validated on the
 * host before any device work), KR_ENONFINITE (NaN / Inf in x or y, counted
 * on the device by the pack / sort kernels), KR_ENOMEM, KR_ECUDA.  Outputs
 * untouched on error.
 * Repeat calls with the same pinned (cudaMallocHost / cudaHostRegister) x, y,
 * h_grid pointers, n, m, kernel and algorithm replay a CUDA graph of the
 * whole call (H2D copies, device pipeline, D2H copies) captured on the first
 * such call; the copies read the buffers' current contents.
 */
int kr_cv_grid(const double *x, const double *y, int64_t n,
               const double *h_grid, int32_t m, int32_t kernel,
               double *cv_out, int32_t *best_out);

/* kr_cv_grid plus the per-bandwidth count of rows with M_i = 1
 * (neff_out [m] int64, nullable). */
int kr_cv_grid_ex(const double *x, const double *y, int64_t n,
                  const double *h_grid, int32_t m, int32_t kernel,
                  double *cv_out, int64_t *neff_out, int32_t *best_out);

/* kr_cv_grid_ex with an explicit algorithm (KR_ALGO_*; KR_EARG if unknown). */
int kr_cv_grid_algo(const double *x, const double *y, int64_t n,
                    const double *h_grid, int32_t m, int32_t kernel, int32_t algo,
                    double *cv_out, int64_t *neff_out, int32_t *best_out);

/*
 * kr_cv_refine -- coarse-to-fine grid search.  §IV.A P@20112-20269: "the
 * user can run the optimization code multiple times with progressively
 * smaller ranges of possible bandwidths".  Level 0 evaluates h_grid[m];
 * level l+1 evaluates m_fine evenly spaced bandwidths on [lo, hi] around level
 * l's best index b (reading Q22): lo = h[b-1] (h[b]/2 if b == 0),
 * hi = h[b+1] (2 h[b] if b is the last index),
 * h_j = lo + (hi - lo) * ((double)j / (m_fine - 1)), h_{m_fine-1} = hi.
 * Levels after the first reuse the device-side sort and prefix moments.
 *   x, y, n, h_grid, m, kernel, algo  as kr_cv_grid_algo (host pointers)
 *   levels       1 .. 64; m_fine 3 .. KR_MAX_M (ignored if levels == 1)
 *   h_best_out   [levels] host: best bandwidth of each level
 *   cv_best_out  [levels] host: its CV
 * Synchronous.  Errors: as kr_cv_grid, KR_EARG for bad levels / m_fine.
 */
int kr_cv_refine(const double *x, const double *y, int64_t n,
                 const double *h_grid, int32_t m, int32_t kernel, int32_t algo,
                 int32_t levels, int32_t m_fine,
                 double *h_best_out, double *cv_best_out);

/*
 * KDE least-squares cross-validation (P@10382-10640: the LSCV machinery
 * "can be applied to ... optimal bandwidth selection for kernel density
 * estimation"; reading Q24).  Kernels normalised to integrate
 * to 1 (uniform, Epanechnikov, triangular; KR_EKERNEL otherwise):
 *   LSCV(h) = int f_h^2 - (2/n) sum_i f_{h,-i}(x_i)
 *           = (n Kbar(0) + sum_i A_i) / (n^2 h) - 2 sum_i B_i / (n (n-1) h),
 *   A_i = sum_{j!=i} Kbar((x_i-x_j)/h) (Kbar = K * K), B_i = sum_{j!=i} K(.)
 * kr_kde_lscv: host pointers, synchronous; lscv_out [m], best_out = smallest
 * arg-min (LSCV may be negative).  Errors: KR_EARG, KR_EKERNEL, KR_EGRID,
 * KR_ENONFINITE, KR_ENOMEM, KR_ECUDA.
 * kr_kde_lscv_async: the same on device pointers, enqueued (workspace from
 * kr_workspace_bytes(n, m)); d_best_status [2] = { best, status }.
 * kr_kde_shard_async: rows [floor(shard n/P), floor((shard+1) n/P)) of the
 * sorted order -> d_partial [KR_PARTIAL_LEN(m)] = [ sum A | sum B | status ],
 * additive across shards; kr_kde_finalize turns the summed partial into LSCV
 * and best on the host (h_grid host pointer).
 */
int kr_kde_lscv(const double *x, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
                double *lscv_out, int32_t *best_out);
int kr_kde_lscv_async(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                      double *d_lscv, int32_t *d_best_status,
                      void *d_workspace, size_t workspace_bytes, void *cuda_stream);
int kr_kde_shard_async(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                       int32_t shard, int32_t nshards, double *d_partial,
                       void *d_workspace, size_t workspace_bytes, void *cuda_stream);
int kr_kde_finalize(const double *partial, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
                    double *lscv_out, int32_t *best_out);

/*
 * Local-linear leave-one-out CV (§IV P@15728-15905: "The
 * Nadaraya-Watson local constant estimator is used rather than a local
 * linear regression" -- the named alternative; reading Q25).
 * Per row i and bandwidth h the LOO estimate is the intercept at x_i of the
 * kernel-weighted least-squares line through the window of Eq.(2) (reading
 * Q1, row i excluded), weights K(|x_l - x_i|/h) of Eq.(3) / footnote 1:
 *   g = (S2 T0 - S1 T1) / (S0 S2 - S1^2),  S_k = sum w d^k, T_k = sum w y d^k.
 * M_i = [the window holds >= 2 distinct x] (else the 2x2 system is
 * singular); CV(h) = n^-1 sum_i M_i (y_i - g)^2 as Eq.(1), best as Q11.
 * Kernels KR_UNIFORM | KR_EPANECHNIKOV | KR_TRIANGULAR (KR_EKERNEL for
 * KR_GAUSSIAN); always the window-prefix path.
 * kr_ll_cv_grid: host pointers, synchronous, outputs as kr_cv_grid_ex
 *   (neff_out nullable).  Errors as kr_cv_grid.
 * kr_ll_cv_grid_async: device pointers, enqueued on cuda_stream; workspace
 *   from kr_workspace_bytes(n, m); d_cv [m], d_neff [m] int64 (nullable),
 *   d_best_status [2] = { best, status }.
 * kr_ll_shard_async: rows [floor(shard n/P), floor((shard+1) n/P)) of the
 *   sorted order -> d_partial [KR_PARTIAL_LEN(m)], the same additive layout
 *   as kr_cv_shard_async, so kr_finalize / kr_finalize_async apply.
 */
int kr_ll_cv_grid(const double *x, const double *y, int64_t n,
                  const double *h_grid, int32_t m, int32_t kernel,
                  double *cv_out, int64_t *neff_out, int32_t *best_out);
int kr_ll_cv_grid_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                        int32_t kernel, double *d_cv, int64_t *d_neff, int32_t *d_best_status,
                        void *d_workspace, size_t workspace_bytes, void *cuda_stream);
int kr_ll_shard_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                      int32_t kernel, int32_t shard, int32_t nshards, double *d_partial,
                      void *d_workspace, size_t workspace_bytes, void *cuda_stream);

/* Host-side grid check (finite, > 0, non-decreasing, 1 <= m <= KR_MAX_M). */
int kr_validate_grid(const double *h_grid, int32_t m);

/* Device workspace size in bytes at (n, m), enough for EVERY device entry
 * point (all algorithms, the KDE family).  Returns 0 for invalid (n, m).
 * Requires a CUDA device (the radix-sort scratch size and the SM count are
 * queried from the runtime). */
size_t kr_workspace_bytes(int64_t n, int32_t m);

/* The workspace one Nadaraya-Watson / local-linear / interval call needs with
 * `algo` (KR_ALGO_*; KR_ALGO_AUTO resolves as the call would) -- the
 * per-algorithm partial-sum blocks only (the split sweep's per-tile partials
 * are the largest; the default window-prefix path needs a few MB per 1,000
 * bandwidths, plus, from n = 50,000 to 2^25, J <= 16 anchored copies of the
 * prefix records at 40 n bytes each -- J = 4 (160 MB) at n = 10^6, DESIGN.md
 * §6.2) -- and the one the KDE entry points need.  An entry point given
 * less than its requirement returns KR_EARG.  0 for invalid (n, m). */
size_t kr_workspace_bytes_algo(int64_t n, int32_t m, int32_t kernel, int32_t algo);
size_t kr_kde_workspace_bytes(int64_t n, int32_t m);

/*
 * kr_cv_shard_async -- device path for caller-owned device memory and row
 * sharding.  Enqueues on `cuda_stream` (a cudaStream_t; NULL = legacy default
 * stream) and returns without synchronising; capturable in a CUDA graph.
 *   d_x, d_y     [n] fp64 DEVICE arrays, unsorted; every shard sees all n
 *   d_h          [m] fp64 DEVICE grid (validate it on the host first with
 *                kr_validate_grid; it is re-checked on the device and a bad
 *                grid is reported through the n_bad_grid slot)
 *   shard, nshards  rows [floor(shard*n/nshards), floor((shard+1)*n/nshards))
 *                of the x-sorted order (stable: ties by original index)
 *   d_partial    [KR_PARTIAL_LEN(m)] fp64 DEVICE output, fully overwritten
 *   d_workspace  >= kr_workspace_bytes(n, m) bytes of device memory, 256-B aligned
 * Host-checked errors (returned): KR_EARG, KR_EKERNEL, KR_ECUDA (launch).
 * Device-detected errors (non-finite x/y, bad device grid) are counted in the
 * status slots and turned into KR_ENONFINITE / KR_EGRID by kr_finalize.
 */
int kr_cv_shard_async(const double *d_x, const double *d_y, int64_t n,
                      const double *d_h, int32_t m, int32_t kernel,
                      int32_t shard, int32_t nshards,
                      double *d_partial, void *d_workspace, size_t workspace_bytes,
                      void *cuda_stream);

/* kr_cv_shard_async with an explicit algorithm (KR_ALGO_*; KR_EARG if
 * unknown).  Same arguments, layout, ownership and errors otherwise. */
int kr_cv_shard_algo_async(const double *d_x, const double *d_y, int64_t n,
                           const double *d_h, int32_t m, int32_t kernel, int32_t algo,
                           int32_t shard, int32_t nshards,
                           double *d_partial, void *d_workspace, size_t workspace_bytes,
                           void *cuda_stream);

/*
 * kr_cv_rows_async -- kr_cv_shard_algo_async for an explicit range of rows:
 * rows [row_lo, row_hi) of the stable x-sorted order (0 <= row_lo <= row_hi
 * <= n, else KR_EARG; an empty range gives a zero partial).  Any set of
 * disjoint ranges covering [0, n) sums to the unsharded partial, so ranks may
 * take unequal row counts of equal cost (cost-balanced
 * partition; the oracle reproduces a range as sorted_rows(x)[lo:hi]).
 * Arguments, layout, ownership and errors otherwise as kr_cv_shard_algo_async.
 */
int kr_cv_rows_async(const double *d_x, const double *d_y, int64_t n,
                     const double *d_h, int32_t m, int32_t kernel, int32_t algo,
                     int64_t row_lo, int64_t row_hi,
                     double *d_partial, void *d_workspace, size_t workspace_bytes,
                     void *cuda_stream);

/*
 * kr_cv_grid_async -- the whole single-GPU grid search on caller-owned device
 * memory, enqueued on `cuda_stream` without synchronising (capturable):
 * kr_cv_shard_algo_async(shard 0 of 1) with the finalize fused into the
 * reduction's last CTA (one launch fewer than shard + kr_finalize_async).
 *   d_x, d_y, d_h, n, m, kernel, algo, d_workspace, workspace_bytes: as
 *                  kr_cv_shard_algo_async (the partial vector lives in the
 *                  workspace)
 *   d_cv           [m] fp64 DEVICE: CV(h_b) per Eq.(1)
 *   d_neff         [m] int64 DEVICE, nullable: rows with M_i = 1 per bandwidth
 *   d_best_status  [2] int32 DEVICE: { best index (Q11), KR_OK | KR_EGRID |
 *                  KR_ENONFINITE } -- read it after the stream work completes
 * Host-checked errors (returned): KR_EARG, KR_EKERNEL, KR_ECUDA.
 */
int kr_cv_grid_async(const double *d_x, const double *d_y, int64_t n,
                     const double *d_h, int32_t m, int32_t kernel, int32_t algo,
                     double *d_cv, int64_t *d_neff, int32_t *d_best_status,
                     void *d_workspace, size_t workspace_bytes, void *cuda_stream);

/*
 * kr_finalize -- host finalize of a partial vector already summed over all
 * shards: cv_out[b] = S[b]/n, neff_out[b] = neff[b] (nullable), best_out per
 * Q11.  Returns KR_EGRID / KR_ENONFINITE if the status slots are non-zero.
 */
int kr_finalize(const double *partial, int64_t n, int32_t m,
                double *cv_out, int64_t *neff_out, int32_t *best_out);

/*
 * kr_finalize_async -- the same on the device (one CTA; the paper's
 * min-reduction kernel, P@24653): d_cv [m] fp64, d_neff [m] int64 (nullable),
 * d_best int32, d_status int32 (KR_OK / KR_EGRID / KR_ENONFINITE).
 */
int kr_finalize_async(const double *d_partial, int64_t n, int32_t m,
                      double *d_cv, int64_t *d_neff, int32_t *d_best, int32_t *d_status,
                      void *cuda_stream);

/*
 * kr_default_grid -- §IV P@16146-16375: max = range of x, min = range/m,
 * evenly spaced; h_b = r * ((double)(b+1)/m), r = max(x) - min(x), so the
 * last point is exactly r (reading Q9).  Host pointers.
 * Errors: KR_EARG, KR_ENONFINITE, KR_EDEGENERATE (r == 0).
 */
int kr_default_grid(const double *x, int64_t n, int32_t m, double *h_out);

/*
 * Leave-one-out cross-validated confidence intervals (§II
 * P@10560-10640: "the estimation of leave-one-out cross-validated confidence
 * intervals for kernel density estimates and kernel regressions"; reading
 * Q26).  Each call runs the grid search first (kr_cv_grid /
 * kr_kde_lscv semantics, same outputs), then at the optimal bandwidth
 * h* = h_grid[best] computes for every observation i (outputs in the caller's
 * order):
 *   kr_cv_ci : est_out[i] = g(x_i), the Nadaraya-Watson estimate from the whole
 *              sample (x_i itself included, Eq.(2) with l = i allowed), and
 *              se_out[i] = the delete-one jackknife standard error
 *              sqrt((n-1)/n sum_j (g^(-j)(x_i) - mean_j g^(-j)(x_i))^2),
 *              g^(-j) the estimate without observation j -- NaN when the
 *              window of x_i holds only x_i (no estimate without it);
 *   kr_kde_ci: est_out[i] = f(x_i) = (1/(n h*)) sum_j K((x_i - x_j)/h*)
 *              (Q24's normalised kernels), se_out[i] its jackknife standard
 *              error, which is the sample standard deviation of the terms
 *              K((x_i - x_j)/h*)/h* over j divided by sqrt(n).
 * The (1 - alpha) interval is est_i -+ z_{1-alpha/2} se_i (the caller's z).
 * Kernels: uniform, Epanechnikov, triangular (the window is compact).
 * Host pointers, synchronous, current CUDA device.  cv_out / lscv_out [m]
 * (the curve of the search), est_out, se_out [n], best_out.
 * Errors: as kr_cv_grid / kr_kde_lscv; KR_EKERNEL for the Gaussian.
 */
int kr_cv_ci(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
             double *cv_out, double *est_out, double *se_out, int32_t *best_out);
int kr_kde_ci(const double *x, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
              double *lscv_out, double *est_out, double *se_out, int32_t *best_out);

/*
 * Device-pointer forms, enqueued on cuda_stream (no host synchronisation:
 * h* is read on the device from the search's best index).  Workspace as
 * kr_cv_grid_async (kr_workspace_bytes(n, m)).  d_cv / d_lscv [m],
 * d_est, d_se [n] fp64, d_best_status [2] int32 {best, status}: read after
 * the stream work completes; est/se are meaningful only if status == KR_OK.
 */
int kr_cv_ci_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                   double *d_cv, double *d_est, double *d_se, int32_t *d_best_status,
                   void *d_workspace, size_t workspace_bytes, void *cuda_stream);
int kr_kde_ci_async(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                    double *d_lscv, double *d_est, double *d_se, int32_t *d_best_status,
                    void *d_workspace, size_t workspace_bytes, void *cuda_stream);

/* Static message for a status code (never NULL). */
const char *kr_strerror(int status);

/* The last CUDA runtime error string seen by this thread ("" if none). */
const char *kr_last_cuda_error(void);

/*
 * Optional stage timing for benchmarks (thread-local state).
 * kr_profile_enable(1): subsequent kr_cv_shard_async calls on this thread
 * record CUDA events on their stream around (a1+a2) pack+sort+gather,
 * the prefix build (window-prefix path only), (a3+a4) the sweep / window
 * kernel and (a5) reduce.  Do not enable while capturing a graph.
 * kr_profile_read waits for the last call's events and writes ms[4]
 * = {sort, prefix_build, sweep, reduce} in milliseconds (prefix_build is ~0
 * on the sweep path); returns KR_EARG if nothing was recorded.
 * kr_launch_count returns the number of kernel launches the last
 * kr_cv_shard_async call on this thread enqueued (CUB passes included);
 * kr_last_algo the algorithm it ran (KR_ALGO_SWEEP or KR_ALGO_PREFIX).
 */
int kr_profile_enable(int on);
int kr_profile_read(float *ms);
int64_t kr_launch_count(void);
int32_t kr_last_algo(void);

/* Library version, e.g. "krcv 0.1.0 sm_100a". */
const char *kr_version(void);

/*
 * kr_release -- frees the state the synchronous host-pointer entry points
 * (kr_cv_grid*, kr_ll_cv_grid, kr_kde_lscv, kr_cv_refine) keep between calls
 * on every device: device buffers, pinned staging, the captured CUDA graph
 * and the library's stream.  The next call re-creates them.  Must not run
 * concurrently with a host call.  Device-pointer (async) calls own no library
 * state and are unaffected.  Returns KR_OK, or KR_ECUDA if a device could
 * not be selected (the others are still released).
 */
int kr_release(void);

#ifdef __cplusplus
}
#endif

#endif /* KRCV_H */
