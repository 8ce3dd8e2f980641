// krcv_host.cpp -- host half of libkrcv.so: validation, default grid, host
// finalize, error strings, and kr_cv_grid (host pointers -> device pipeline
// of krcv_device.cu on a lazily created per-device context).
#include <cuda_runtime.h>

#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "krcv.h"
#include "krcv_internal.h"

namespace krcv {

static thread_local std::string g_last_cuda_error;

void set_cuda_error(const char *what, int code)
{
    char buf[512];
    std::snprintf(buf, sizeof buf, "%s: %s (%d)", what,
                  cudaGetErrorString(static_cast<cudaError_t>(code)), code);
    g_last_cuda_error = buf;
}

static bool kernel_ok(int32_t k)
{
    return k == KR_UNIFORM || k == KR_EPANECHNIKOV || k == KR_TRIANGULAR || k == KR_GAUSSIAN;
}

// Per-device context for the synchronous host-pointer entry point.
struct DevCtx {
    std::mutex mu;
    cudaStream_t stream = nullptr;
    void *ws = nullptr;
    size_t ws_bytes = 0;
    double *dx = nullptr, *dy = nullptr, *dh = nullptr;
    int64_t cap_n = 0;
    int32_t cap_m = 0;
    double *dpartial = nullptr, *dcv = nullptr;
    int64_t *dneff = nullptr;
    int32_t *dbest = nullptr;  // [2]: best, status
};

static std::mutex g_ctx_mu;
static std::vector<DevCtx *> g_ctx;

static DevCtx *get_ctx(int dev)
{
    std::lock_guard<std::mutex> g(g_ctx_mu);
    if ((int)g_ctx.size() <= dev) g_ctx.resize(dev + 1, nullptr);
    if (!g_ctx[dev]) g_ctx[dev] = new DevCtx();  // process lifetime
    return g_ctx[dev];
}

#define KR_CUDA_TRY(call)                                   \
    do {                                                    \
        cudaError_t e_ = (call);                            \
        if (e_ != cudaSuccess) {                            \
            set_cuda_error(#call, (int)e_);                 \
            return e_ == cudaErrorMemoryAllocation ? KR_ENOMEM : KR_ECUDA; \
        }                                                   \
    } while (0)

static int ensure_capacity(DevCtx *c, int64_t n, int32_t m)
{
    if (!c->stream) KR_CUDA_TRY(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
    if (n > c->cap_n) {
        cudaFree(c->dx);
        cudaFree(c->dy);
        c->dx = c->dy = nullptr;
        c->cap_n = 0;
        KR_CUDA_TRY(cudaMalloc(&c->dx, sizeof(double) * n));
        KR_CUDA_TRY(cudaMalloc(&c->dy, sizeof(double) * n));
        c->cap_n = n;
    }
    if (m > c->cap_m) {
        cudaFree(c->dh);
        cudaFree(c->dpartial);
        cudaFree(c->dcv);
        cudaFree(c->dneff);
        cudaFree(c->dbest);
        c->dh = c->dpartial = c->dcv = nullptr;
        c->dneff = nullptr;
        c->dbest = nullptr;
        c->cap_m = 0;
        KR_CUDA_TRY(cudaMalloc(&c->dh, sizeof(double) * m));
        KR_CUDA_TRY(cudaMalloc(&c->dpartial, sizeof(double) * KR_PARTIAL_LEN(m)));
        KR_CUDA_TRY(cudaMalloc(&c->dcv, sizeof(double) * m));
        KR_CUDA_TRY(cudaMalloc(&c->dneff, sizeof(int64_t) * m));
        KR_CUDA_TRY(cudaMalloc(&c->dbest, sizeof(int32_t) * 2));
        c->cap_m = m;
    }
    size_t need = kr_workspace_bytes(n, m);
    if (need == 0) return KR_ECUDA;
    if (need > c->ws_bytes) {
        cudaFree(c->ws);
        c->ws = nullptr;
        c->ws_bytes = 0;
        KR_CUDA_TRY(cudaMalloc(&c->ws, need));
        c->ws_bytes = need;
    }
    return KR_OK;
}

}  // namespace krcv

using namespace krcv;

extern "C" int kr_validate_grid(const double *h, int32_t m)
{
    if (!h || m < 1 || m > KR_MAX_M) return KR_EARG;
    for (int32_t b = 0; b < m; b++) {
        if (!std::isfinite(h[b]) || !(h[b] > 0.0)) return KR_EGRID;
        if (b > 0 && h[b] < h[b - 1]) return KR_EGRID;
    }
    return KR_OK;
}

static int validate_all(const double *x, const double *y, int64_t n, const double *h, int32_t m,
                        int32_t kernel)
{
    if (!x || !y || !h) return KR_EARG;
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (!kernel_ok(kernel)) return KR_EKERNEL;
    int st = kr_validate_grid(h, m);
    if (st) return st;
    for (int64_t i = 0; i < n; i++)
        if (!std::isfinite(x[i]) || !std::isfinite(y[i])) return KR_ENONFINITE;
    return KR_OK;
}

extern "C" int kr_cv_grid_algo(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                               int32_t kernel, int32_t algo, double *cv_out, int64_t *neff_out,
                               int32_t *best_out)
{
    if (!cv_out || !best_out) return KR_EARG;
    if (algo != KR_ALGO_AUTO && algo != KR_ALGO_SWEEP && algo != KR_ALGO_PREFIX && algo != KR_ALGO_DENSE &&
        algo != KR_ALGO_HIST)
        return KR_EARG;
    int st = validate_all(x, y, n, h_grid, m, kernel);
    if (st) return st;
    int dev = 0;
    KR_CUDA_TRY(cudaGetDevice(&dev));
    DevCtx *c = get_ctx(dev);
    std::lock_guard<std::mutex> g(c->mu);
    st = ensure_capacity(c, n, m);
    if (st) return st;
    cudaStream_t s = c->stream;
    KR_CUDA_TRY(cudaMemcpyAsync(c->dx, x, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dy, y, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dh, h_grid, sizeof(double) * m, cudaMemcpyHostToDevice, s));
    st = kr_cv_grid_async(c->dx, c->dy, n, c->dh, m, kernel, algo, c->dcv, c->dneff, c->dbest, c->ws, c->ws_bytes,
                          s);
    if (st) return st;
    std::vector<double> cv(m);
    std::vector<int64_t> ne(neff_out ? m : 0);
    int32_t bs[2] = {0, 0};
    KR_CUDA_TRY(cudaMemcpyAsync(cv.data(), c->dcv, sizeof(double) * m, cudaMemcpyDeviceToHost, s));
    if (neff_out)
        KR_CUDA_TRY(cudaMemcpyAsync(ne.data(), c->dneff, sizeof(int64_t) * m, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaMemcpyAsync(bs, c->dbest, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaStreamSynchronize(s));
    if (bs[1] != KR_OK) return bs[1];
    std::memcpy(cv_out, cv.data(), sizeof(double) * m);
    if (neff_out) std::memcpy(neff_out, ne.data(), sizeof(int64_t) * m);
    *best_out = bs[0];
    return KR_OK;
}

extern "C" int kr_ll_cv_grid(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                             int32_t kernel, double *cv_out, int64_t *neff_out, int32_t *best_out)
{
    if (!cv_out || !best_out) return KR_EARG;
    int st = validate_all(x, y, n, h_grid, m, kernel);
    if (st) return st;
    if (kernel == KR_GAUSSIAN) return KR_EKERNEL;
    int dev = 0;
    KR_CUDA_TRY(cudaGetDevice(&dev));
    DevCtx *c = get_ctx(dev);
    std::lock_guard<std::mutex> g(c->mu);
    st = ensure_capacity(c, n, m);
    if (st) return st;
    cudaStream_t s = c->stream;
    KR_CUDA_TRY(cudaMemcpyAsync(c->dx, x, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dy, y, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dh, h_grid, sizeof(double) * m, cudaMemcpyHostToDevice, s));
    st = kr_ll_cv_grid_async(c->dx, c->dy, n, c->dh, m, kernel, c->dcv, c->dneff, c->dbest, c->ws, c->ws_bytes, s);
    if (st) return st;
    std::vector<double> cv(m);
    std::vector<int64_t> ne(neff_out ? m : 0);
    int32_t bs[2] = {0, 0};
    KR_CUDA_TRY(cudaMemcpyAsync(cv.data(), c->dcv, sizeof(double) * m, cudaMemcpyDeviceToHost, s));
    if (neff_out)
        KR_CUDA_TRY(cudaMemcpyAsync(ne.data(), c->dneff, sizeof(int64_t) * m, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaMemcpyAsync(bs, c->dbest, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaStreamSynchronize(s));
    if (bs[1] != KR_OK) return bs[1];
    std::memcpy(cv_out, cv.data(), sizeof(double) * m);
    if (neff_out) std::memcpy(neff_out, ne.data(), sizeof(int64_t) * m);
    *best_out = bs[0];
    return KR_OK;
}

extern "C" int kr_cv_grid_ex(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                             int32_t kernel, double *cv_out, int64_t *neff_out, int32_t *best_out)
{
    return kr_cv_grid_algo(x, y, n, h_grid, m, kernel, KR_ALGO_AUTO, cv_out, neff_out, best_out);
}

extern "C" int kr_cv_grid(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                          int32_t kernel, double *cv_out, int32_t *best_out)
{
    return kr_cv_grid_ex(x, y, n, h_grid, m, kernel, cv_out, nullptr, best_out);
}

// Level l+1's grid around level l's best index (reading Q22):
// [lo, hi] = [h[b-1], h[b+1]] (h[b]/2 below the first, 2 h[b] above the
// last point), m_fine evenly spaced points with both ends included.
static void refine_grid(const std::vector<double> &h, int32_t best, int32_t m_fine, std::vector<double> &out)
{
    const int32_t m = (int32_t)h.size();
    const double lo = best > 0 ? h[best - 1] : h[best] / 2.0;
    const double hi = best < m - 1 ? h[best + 1] : 2.0 * h[best];
    out.resize(m_fine);
    const double w = hi - lo;
    for (int32_t j = 0; j < m_fine; j++) {
        const double t = (double)j / (double)(m_fine - 1);
        const double p = w * t;
        out[j] = lo + p;
    }
    out[m_fine - 1] = hi;
}

extern "C" int kr_cv_refine(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                            int32_t kernel, int32_t algo, int32_t levels, int32_t m_fine, double *h_best_out,
                            double *cv_best_out)
{
    if (!h_best_out || !cv_best_out || levels < 1 || levels > 64) return KR_EARG;
    if (levels > 1 && (m_fine < 3 || m_fine > KR_MAX_M)) return KR_EARG;
    if (algo != KR_ALGO_AUTO && algo != KR_ALGO_SWEEP && algo != KR_ALGO_PREFIX && algo != KR_ALGO_DENSE &&
        algo != KR_ALGO_HIST)
        return KR_EARG;
    int st = validate_all(x, y, n, h_grid, m, kernel);
    if (st) return st;
    int dev = 0;
    KR_CUDA_TRY(cudaGetDevice(&dev));
    DevCtx *c = get_ctx(dev);
    std::lock_guard<std::mutex> g(c->mu);
    const int32_t mcap = levels > 1 && m_fine > m ? m_fine : m;
    st = ensure_capacity(c, n, mcap);
    if (st) return st;
    cudaStream_t s = c->stream;
    KR_CUDA_TRY(cudaMemcpyAsync(c->dx, x, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dy, y, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    std::vector<double> h(h_grid, h_grid + m), next, cv;
    for (int32_t l = 0; l < levels; l++) {
        const int32_t ml = (int32_t)h.size();
        st = kr_validate_grid(h.data(), ml);
        if (st) return st;  // a refined grid of a degenerate level (lo == hi) is still valid
        KR_CUDA_TRY(cudaMemcpyAsync(c->dh, h.data(), sizeof(double) * ml, cudaMemcpyHostToDevice, s));
        // level 0 sorts and builds the prefix moments; later levels reuse them
        st = enqueue_grid(c->dx, c->dy, n, c->dh, ml, kernel, algo, c->dcv, nullptr, c->dbest, c->ws, c->ws_bytes,
                          s, l > 0);
        if (st) return st;
        cv.resize(ml);
        int32_t bs[2] = {0, 0};
        KR_CUDA_TRY(cudaMemcpyAsync(cv.data(), c->dcv, sizeof(double) * ml, cudaMemcpyDeviceToHost, s));
        KR_CUDA_TRY(cudaMemcpyAsync(bs, c->dbest, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
        KR_CUDA_TRY(cudaStreamSynchronize(s));
        if (bs[1] != KR_OK) return bs[1];
        h_best_out[l] = h[bs[0]];
        cv_best_out[l] = cv[bs[0]];
        if (l + 1 < levels) {
            refine_grid(h, bs[0], m_fine, next);
            h.swap(next);
        }
    }
    return KR_OK;
}

extern "C" int kr_kde_lscv(const double *x, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
                           double *lscv_out, int32_t *best_out)
{
    if (!x || !h_grid || !lscv_out || !best_out) return KR_EARG;
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (kernel != KR_UNIFORM && kernel != KR_EPANECHNIKOV && kernel != KR_TRIANGULAR) return KR_EKERNEL;
    int st = kr_validate_grid(h_grid, m);
    if (st) return st;
    for (int64_t i = 0; i < n; i++)
        if (!std::isfinite(x[i])) return KR_ENONFINITE;
    int dev = 0;
    KR_CUDA_TRY(cudaGetDevice(&dev));
    DevCtx *c = get_ctx(dev);
    std::lock_guard<std::mutex> g(c->mu);
    st = ensure_capacity(c, n, m);
    if (st) return st;
    cudaStream_t s = c->stream;
    KR_CUDA_TRY(cudaMemcpyAsync(c->dx, x, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dh, h_grid, sizeof(double) * m, cudaMemcpyHostToDevice, s));
    st = kr_kde_lscv_async(c->dx, n, c->dh, m, kernel, c->dcv, c->dbest, c->ws, c->ws_bytes, s);
    if (st) return st;
    std::vector<double> v(m);
    int32_t bs[2] = {0, 0};
    KR_CUDA_TRY(cudaMemcpyAsync(v.data(), c->dcv, sizeof(double) * m, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaMemcpyAsync(bs, c->dbest, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaStreamSynchronize(s));
    if (bs[1] != KR_OK) return bs[1];
    std::memcpy(lscv_out, v.data(), sizeof(double) * m);
    *best_out = bs[0];
    return KR_OK;
}

extern "C" int kr_kde_finalize(const double *partial, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
                               double *lscv_out, int32_t *best_out)
{
    if (!partial || !h_grid || !lscv_out || !best_out || n < 2 || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (kernel != KR_UNIFORM && kernel != KR_EPANECHNIKOV && kernel != KR_TRIANGULAR) return KR_EKERNEL;
    if (partial[2 * (int64_t)m] != 0.0) return KR_EGRID;
    if (partial[2 * (int64_t)m + 1] != 0.0) return KR_ENONFINITE;
    const double nn = (double)n;
    const double kb0 = kernel == KR_UNIFORM ? 0.5 : (kernel == KR_EPANECHNIKOV ? 0.6 : 2.0 / 3.0);
    int32_t best = -1;
    double bv = 0.0;
    for (int32_t b = 0; b < m; b++) {
        const double v = (nn * kb0 + partial[b]) / (nn * nn * h_grid[b]) -
                         2.0 * partial[m + b] / (nn * (nn - 1.0) * h_grid[b]);
        lscv_out[b] = v;
        if (!std::isnan(v) && (best < 0 || v < bv)) {
            bv = v;
            best = b;
        }
    }
    *best_out = best < 0 ? 0 : best;
    return KR_OK;
}

extern "C" int kr_finalize(const double *partial, int64_t n, int32_t m, double *cv_out, int64_t *neff_out,
                           int32_t *best_out)
{
    if (!partial || !cv_out || !best_out || n < 1 || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (partial[2 * (int64_t)m] != 0.0) return KR_EGRID;
    if (partial[2 * (int64_t)m + 1] != 0.0) return KR_ENONFINITE;
    int32_t best = -1;
    double bv = 0.0;
    for (int32_t b = 0; b < m; b++) {
        double v = partial[b] / (double)n;  // Eq.(1): n^-1 sum_i
        cv_out[b] = v;
        if (neff_out) neff_out[b] = (int64_t)partial[m + b];
        if (!std::isnan(v) && (best < 0 || v < bv)) {  // Q11: first minimum
            bv = v;
            best = b;
        }
    }
    *best_out = best < 0 ? 0 : best;
    return KR_OK;
}

extern "C" int kr_default_grid(const double *x, int64_t n, int32_t m, double *h_out)
{
    if (!x || !h_out || n < 2 || m < 1 || m > KR_MAX_M) return KR_EARG;
    double lo = x[0], hi = x[0];
    for (int64_t i = 0; i < n; i++) {
        if (!std::isfinite(x[i])) return KR_ENONFINITE;
        lo = x[i] < lo ? x[i] : lo;
        hi = x[i] > hi ? x[i] : hi;
    }
    const double r = hi - lo;  // "the domain of X_i" P@16146
    if (!(r > 0.0)) return KR_EDEGENERATE;
    for (int32_t b = 0; b < m; b++) h_out[b] = r * ((double)(b + 1) / (double)m);
    return KR_OK;
}

extern "C" const char *kr_strerror(int status)
{
    switch (status) {
    case KR_OK: return "ok";
    case KR_EARG: return "invalid argument (null pointer, size out of range, bad shard or workspace)";
    case KR_EKERNEL: return "unknown kernel";
    case KR_EGRID: return "bandwidth grid must be finite, > 0 and non-decreasing";
    case KR_ENONFINITE: return "x or y contains NaN or Inf";
    case KR_EDEGENERATE: return "degenerate data: max(x) == min(x)";
    case KR_ENOMEM: return "out of memory";
    case KR_ECUDA: return "CUDA runtime error (see kr_last_cuda_error)";
    default: return "unknown status";
    }
}

extern "C" const char *kr_last_cuda_error(void) { return g_last_cuda_error.c_str(); }

extern "C" const char *kr_version(void) { return "krcv 0.1.0 sm_100a"; }
