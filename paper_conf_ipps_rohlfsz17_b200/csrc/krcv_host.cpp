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

void set_error_text(const char *text) { g_last_cuda_error = text; }

static bool kernel_ok(int32_t k)
{
    return k == KR_UNIFORM || k == KR_EPANECHNIKOV || k == KR_TRIANGULAR || k == KR_GAUSSIAN;
}

// Per-device context for the synchronous host-pointer entry point.
struct DevCtx {
    std::mutex mu;
    cudaStream_t stream = nullptr;
    // side streams and events that fork the three input copies into parallel
    // branches (x on `stream`, y and h on side[0], side[1]) and join them
    cudaStream_t side[2] = {nullptr, nullptr};
    cudaEvent_t ev_fork = nullptr, ev_join[2] = {nullptr, nullptr};
    void *ws = nullptr;
    size_t ws_bytes = 0;
    double *dx = nullptr, *dy = nullptr, *dh = nullptr;
    int64_t cap_n = 0;
    int32_t cap_m = 0;
    double *dpartial = nullptr;
    // results of the synchronous host path, one block [best, status | cv[m] |
    // neff[m]] on the device (refinement, KDE) and its pinned mapped mirror, which
    // the finalize of kr_cv_grid* / kr_ll_cv_grid writes directly (no D2H copy)
    char *dres = nullptr;
    double *dcv = nullptr;
    int64_t *dneff = nullptr;
    int32_t *dbest = nullptr;  // [2]: best, status
    char *pres = nullptr;
    int32_t pcap_m = 0;
    // CUDA graph of the last synchronous call whose inputs were pinned
    // (H2D copies, the whole device pipeline, D2H copies): replayed while
    // the pointers, sizes, kernel, algorithm and estimator repeat
    // confidence-interval outputs [n] (kr_cv_ci / kr_kde_ci)
    double *dest = nullptr, *dse = nullptr;
    int64_t cap_ci = 0;
    cudaGraphExec_t gexec = nullptr;
    const void *gx = nullptr, *gy = nullptr, *gh = nullptr;
    int64_t gn = 0;
    int32_t gm = 0, gkernel = -1, galgo = -1, gll = -1;
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

// The captured host-path graph (DevCtx::gexec) has c->dx, c->dy, c->dh,
// c->ws and the pinned staging c->pres baked into its nodes: any
// reallocation of one of them must drop it, or a later replay with the same
// caller pointers would copy into / launch on freed memory.
static void drop_graph(DevCtx *c)
{
    if (c->gexec) cudaGraphExecDestroy(c->gexec);
    c->gexec = nullptr;
    c->gx = c->gy = c->gh = nullptr;
}

// [best, status] (8 B) | cv[m] | neff[m]
static size_t res_bytes(int32_t m) { return 8 + (sizeof(double) + sizeof(int64_t)) * (size_t)m; }

static int ensure_capacity(DevCtx *c, int64_t n, int32_t m, size_t need)
{
    if (!c->stream) {
        KR_CUDA_TRY(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking));
        for (int i = 0; i < 2; i++) {
            KR_CUDA_TRY(cudaStreamCreateWithFlags(&c->side[i], cudaStreamNonBlocking));
            KR_CUDA_TRY(cudaEventCreateWithFlags(&c->ev_join[i], cudaEventDisableTiming));
        }
        KR_CUDA_TRY(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
    }
    if (n > c->cap_n) {
        drop_graph(c);
        cudaFree(c->dx);
        cudaFree(c->dy);
        c->dx = c->dy = nullptr;
        c->cap_n = 0;
        KR_CUDA_TRY(cudaMalloc(&c->dx, sizeof(double) * n));
        KR_CUDA_TRY(cudaMalloc(&c->dy, sizeof(double) * n));
        c->cap_n = n;
    }
    if (m > c->cap_m) {
        drop_graph(c);
        cudaFree(c->dh);
        cudaFree(c->dpartial);
        cudaFree(c->dres);
        c->dh = c->dpartial = c->dcv = nullptr;
        c->dres = nullptr;
        c->dneff = nullptr;
        c->dbest = nullptr;
        c->cap_m = 0;
        KR_CUDA_TRY(cudaMalloc(&c->dh, sizeof(double) * m));
        KR_CUDA_TRY(cudaMalloc(&c->dpartial, sizeof(double) * KR_PARTIAL_LEN(m)));
        KR_CUDA_TRY(cudaMalloc(&c->dres, res_bytes(m)));
        c->dbest = reinterpret_cast<int32_t *>(c->dres);
        c->dcv = reinterpret_cast<double *>(c->dres + 8);
        c->dneff = reinterpret_cast<int64_t *>(c->dres + 8 + sizeof(double) * m);
        c->cap_m = m;
    }
    if (need == 0) return KR_ECUDA;
    if (need > c->ws_bytes) {
        drop_graph(c);
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
    // x, y are checked for NaN / Inf on the device (the pack / chunk-sort
    // kernels count them into the status word, and the call returns
    // KR_ENONFINITE with the outputs untouched): a host scan would cost more
    // than the whole C2 search's H2D copy
    return kr_validate_grid(h, m);
}

static bool is_pinned(const void *p)
{
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeHost;
}

static int ensure_staging(DevCtx *c, int32_t m)
{
    if (m <= c->pcap_m) return KR_OK;
    drop_graph(c);
    cudaFreeHost(c->pres);
    c->pres = nullptr;
    c->pcap_m = 0;
    KR_CUDA_TRY(cudaMallocHost(&c->pres, res_bytes(m)));
    c->pcap_m = m;
    return KR_OK;
}

// H2D of the inputs, the whole device search (Nadaraya-Watson or
// local-linear), D2H of the results into the pinned staging -- all enqueued
// on c->stream.
static int enqueue_host_call(DevCtx *c, const double *x, const double *y, int64_t n, const double *h, int32_t m,
                             int32_t kernel, int32_t algo, bool ll)
{
    cudaStream_t s = c->stream;
    // the three input copies run as parallel branches (one copy engine each)
    KR_CUDA_TRY(cudaEventRecord(c->ev_fork, s));
    for (int i = 0; i < 2; i++) KR_CUDA_TRY(cudaStreamWaitEvent(c->side[i], c->ev_fork, 0));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dx, x, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dy, y, sizeof(double) * n, cudaMemcpyHostToDevice, c->side[0]));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dh, h, sizeof(double) * m, cudaMemcpyHostToDevice, c->side[1]));
    for (int i = 0; i < 2; i++) {
        KR_CUDA_TRY(cudaEventRecord(c->ev_join[i], c->side[i]));
        KR_CUDA_TRY(cudaStreamWaitEvent(s, c->ev_join[i], 0));
    }
    // the finalize (fused into the reduction's last CTA) writes the result
    // block -- [best, status | cv[m] | neff[m]] laid out for this call's m --
    // straight into the mapped pinned staging: no device-to-host copy
    char *pres = nullptr;
    KR_CUDA_TRY(cudaHostGetDevicePointer(reinterpret_cast<void **>(&pres), c->pres, 0));
    int32_t *dbest = reinterpret_cast<int32_t *>(pres);
    double *dcv = reinterpret_cast<double *>(pres + 8);
    int64_t *dneff = reinterpret_cast<int64_t *>(pres + 8 + sizeof(double) * m);
    const int st = ll ? kr_ll_cv_grid_async(c->dx, c->dy, n, c->dh, m, kernel, dcv, dneff, dbest, c->ws,
                                            c->ws_bytes, s)
                      : kr_cv_grid_async(c->dx, c->dy, n, c->dh, m, kernel, algo, dcv, dneff, dbest, c->ws,
                                         c->ws_bytes, s);
    if (st) return st;
    return KR_OK;
}

// The synchronous host-pointer path shared by kr_cv_grid* and kr_ll_cv_grid.
// With pinned x, y, h (and profiling off) the enqueued sequence is captured
// once as a CUDA graph and replayed on repeat calls -- one launch instead of
// ~13 API calls; the copies read the caller's buffers at replay time.
static int host_call(const double *x, const double *y, int64_t n, const double *h, int32_t m, int32_t kernel,
                     int32_t algo, bool ll, double *cv_out, int64_t *neff_out, int32_t *best_out)
{
    int dev = 0;
    KR_CUDA_TRY(cudaGetDevice(&dev));
    DevCtx *c = get_ctx(dev);
    std::lock_guard<std::mutex> g(c->mu);
    int st = ensure_capacity(c, n, m, ll ? kr_workspace_bytes_algo(n, m, kernel, KR_ALGO_PREFIX)
                                         : kr_workspace_bytes_algo(n, m, kernel, algo));
    if (st) return st;
    st = ensure_staging(c, m);
    if (st) return st;
    cudaStream_t s = c->stream;
    const bool graph = !prof_enabled() && is_pinned(x) && is_pinned(y) && is_pinned(h);
    if (graph) {
        const bool same = c->gexec && c->gx == x && c->gy == y && c->gh == h && c->gn == n && c->gm == m &&
                          c->gkernel == kernel && c->galgo == algo && c->gll == (ll ? 1 : 0);
        if (!same) {
            if (c->gexec) cudaGraphExecDestroy(c->gexec);
            c->gexec = nullptr;
            KR_CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
            st = enqueue_host_call(c, x, y, n, h, m, kernel, algo, ll);
            cudaGraph_t gr = nullptr;
            const cudaError_t e = cudaStreamEndCapture(s, &gr);
            if (st) {
                if (gr) cudaGraphDestroy(gr);
                return st;
            }
            if (e != cudaSuccess) {
                set_cuda_error("cudaStreamEndCapture", (int)e);
                return KR_ECUDA;
            }
            const cudaError_t e2 = cudaGraphInstantiate(&c->gexec, gr, 0);
            cudaGraphDestroy(gr);
            if (e2 != cudaSuccess) {
                c->gexec = nullptr;
                set_cuda_error("cudaGraphInstantiate", (int)e2);
                return KR_ECUDA;
            }
            c->gx = x;
            c->gy = y;
            c->gh = h;
            c->gn = n;
            c->gm = m;
            c->gkernel = kernel;
            c->galgo = algo;
            c->gll = ll ? 1 : 0;
        }
        KR_CUDA_TRY(cudaGraphLaunch(c->gexec, s));
    } else {
        st = enqueue_host_call(c, x, y, n, h, m, kernel, algo, ll);
        if (st) return st;
    }
    KR_CUDA_TRY(cudaStreamSynchronize(s));
    const int32_t *pbs = reinterpret_cast<const int32_t *>(c->pres);  // layout of enqueue_host_call
    if (pbs[1] != KR_OK) return pbs[1];
    std::memcpy(cv_out, c->pres + 8, sizeof(double) * m);
    if (neff_out) std::memcpy(neff_out, c->pres + 8 + sizeof(double) * m, sizeof(int64_t) * m);
    *best_out = pbs[0];
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
    const int st = validate_all(x, y, n, h_grid, m, kernel);
    if (st) return st;
    return host_call(x, y, n, h_grid, m, kernel, algo, false, cv_out, neff_out, best_out);
}

extern "C" int kr_ll_cv_grid(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                             int32_t kernel, double *cv_out, int64_t *neff_out, int32_t *best_out)
{
    if (!cv_out || !best_out) return KR_EARG;
    const int st = validate_all(x, y, n, h_grid, m, kernel);
    if (st) return st;
    if (kernel == KR_GAUSSIAN) return KR_EKERNEL;
    return host_call(x, y, n, h_grid, m, kernel, KR_ALGO_PREFIX, true, cv_out, neff_out, best_out);
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
    st = ensure_capacity(c, n, mcap, kr_workspace_bytes_algo(n, mcap, kernel, algo));
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
    st = ensure_capacity(c, n, m, kr_kde_workspace_bytes(n, m));
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

// Leave-one-out (jackknife) confidence intervals at the CV / LSCV optimum
// (reading Q26): the device search, the interval kernel, one copy back.
static int host_ci(bool kde, const double *x, const double *y, int64_t n, const double *h_grid, int32_t m,
                   int32_t kernel, double *curve_out, double *est_out, double *se_out, int32_t *best_out)
{
    if (!curve_out || !est_out || !se_out || !best_out) return KR_EARG;
    int st = kde ? (x && h_grid ? KR_OK : KR_EARG) : validate_all(x, y, n, h_grid, m, kernel);
    if (st) return st;
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (kernel != KR_UNIFORM && kernel != KR_EPANECHNIKOV && kernel != KR_TRIANGULAR) return KR_EKERNEL;
    if (kde) {
        st = kr_validate_grid(h_grid, m);
        if (st) return st;
        for (int64_t i = 0; i < n; i++)
            if (!std::isfinite(x[i])) return KR_ENONFINITE;
    }
    int dev = 0;
    KR_CUDA_TRY(cudaGetDevice(&dev));
    DevCtx *c = get_ctx(dev);
    std::lock_guard<std::mutex> g(c->mu);
    st = ensure_capacity(c, n, m, kde ? kr_kde_workspace_bytes(n, m) : kr_workspace_bytes_algo(n, m, kernel, KR_ALGO_AUTO));
    if (st) return st;
    if (n > c->cap_ci) {
        cudaFree(c->dest);
        cudaFree(c->dse);
        c->dest = c->dse = nullptr;
        c->cap_ci = 0;
        KR_CUDA_TRY(cudaMalloc(&c->dest, sizeof(double) * n));
        KR_CUDA_TRY(cudaMalloc(&c->dse, sizeof(double) * n));
        c->cap_ci = n;
    }
    cudaStream_t s = c->stream;
    KR_CUDA_TRY(cudaMemcpyAsync(c->dx, x, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    if (!kde) KR_CUDA_TRY(cudaMemcpyAsync(c->dy, y, sizeof(double) * n, cudaMemcpyHostToDevice, s));
    KR_CUDA_TRY(cudaMemcpyAsync(c->dh, h_grid, sizeof(double) * m, cudaMemcpyHostToDevice, s));
    st = kde ? kr_kde_ci_async(c->dx, n, c->dh, m, kernel, c->dcv, c->dest, c->dse, c->dbest, c->ws, c->ws_bytes, s)
             : kr_cv_ci_async(c->dx, c->dy, n, c->dh, m, kernel, c->dcv, c->dest, c->dse, c->dbest, c->ws,
                              c->ws_bytes, s);
    if (st) return st;
    int32_t bs[2] = {0, 0};
    KR_CUDA_TRY(cudaMemcpyAsync(bs, c->dbest, sizeof(int32_t) * 2, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaMemcpyAsync(curve_out, c->dcv, sizeof(double) * m, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaMemcpyAsync(est_out, c->dest, sizeof(double) * n, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaMemcpyAsync(se_out, c->dse, sizeof(double) * n, cudaMemcpyDeviceToHost, s));
    KR_CUDA_TRY(cudaStreamSynchronize(s));
    if (bs[1] != KR_OK) return bs[1];
    *best_out = bs[0];
    return KR_OK;
}

extern "C" int kr_cv_ci(const double *x, const double *y, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
                        double *cv_out, double *est_out, double *se_out, int32_t *best_out)
{
    return host_ci(false, x, y, n, h_grid, m, kernel, cv_out, est_out, se_out, best_out);
}

extern "C" int kr_kde_ci(const double *x, int64_t n, const double *h_grid, int32_t m, int32_t kernel,
                         double *lscv_out, double *est_out, double *se_out, int32_t *best_out)
{
    return host_ci(true, x, nullptr, n, h_grid, m, kernel, lscv_out, est_out, se_out, best_out);
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

// Frees what the synchronous host entry points keep between calls on every
// device (buffers, pinned staging, the captured graph, the stream); the next
// call re-creates them.  The caller must not have a host call in flight.
extern "C" int kr_release(void)
{
    std::lock_guard<std::mutex> g(g_ctx_mu);
    int prev = 0;
    cudaGetDevice(&prev);
    int st = KR_OK;
    for (size_t d = 0; d < g_ctx.size(); d++) {
        DevCtx *c = g_ctx[d];
        if (!c) continue;
        std::lock_guard<std::mutex> lk(c->mu);
        if (cudaSetDevice((int)d) != cudaSuccess) { st = KR_ECUDA; continue; }
        if (c->stream) cudaStreamSynchronize(c->stream);
        if (c->gexec) cudaGraphExecDestroy(c->gexec);
        cudaFree(c->ws);
        cudaFree(c->dx);
        cudaFree(c->dy);
        cudaFree(c->dh);
        cudaFree(c->dpartial);
        cudaFree(c->dres);
        cudaFree(c->dest);
        cudaFree(c->dse);
        c->dest = c->dse = nullptr;
        c->cap_ci = 0;
        cudaFreeHost(c->pres);
        if (c->stream) cudaStreamDestroy(c->stream);
        for (int i = 0; i < 2; i++) {
            if (c->side[i]) cudaStreamDestroy(c->side[i]);
            if (c->ev_join[i]) cudaEventDestroy(c->ev_join[i]);
            c->side[i] = nullptr;
            c->ev_join[i] = nullptr;
        }
        if (c->ev_fork) cudaEventDestroy(c->ev_fork);
        c->ev_fork = nullptr;
        c->gexec = nullptr;
        c->gx = c->gy = c->gh = nullptr;
        c->ws = nullptr;
        c->ws_bytes = 0;
        c->dx = c->dy = c->dh = c->dpartial = c->dcv = nullptr;
        c->dres = nullptr;
        c->dneff = nullptr;
        c->dbest = nullptr;
        c->pres = nullptr;
        c->pcap_m = 0;
        c->cap_n = 0;
        c->cap_m = 0;
        c->stream = nullptr;
    }
    cudaSetDevice(prev);
    return st;
}
