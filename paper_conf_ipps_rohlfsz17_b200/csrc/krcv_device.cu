// krcv_device.cu -- sm_100a kernels of the LOO-CV bandwidth grid search and
// the device half of the C-ABI (kr_workspace_bytes, kr_cv_shard_async,
// kr_finalize_async).  See include/krcv.h and DESIGN.md.
//
// Hot path, one pass per call:
//   a1 pack      x -> order-preserving uint64 key, index; validity counters
//   a2 sort      CUB onesweep radix sort of (key, index), stable; gather (x,y)
//   a3 sweep     per sorted row: fused distance + window test + running sums,
//                bandwidths ascending (§III P@14010-14984,
//                §IV.B P@21154-22104), realised on the globally sorted array:
//                row i's right neighbours i+1, i+2, ... and left neighbours
//                i-1, i-2, ... are already in increasing |x_l - x_i| order.
//   a4 emit      LOO estimate Eq.(2), M, squared error Eq.(1) per (row, h_b)
//   a5 reduce    per-warp-tile partials -> fixed-order column sums -> partial
// All arithmetic fp64; no tensor cores (not a contraction).
#include <cuda_runtime.h>
#include <cub/device/device_radix_sort.cuh>

#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

#include "krcv.h"
#include <nvtx3/nvToolsExt.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>
#include "krcv_internal.h"
#include "krcv_pdl.cuh"
#include "krcv_sweep.cuh"
#include "krcv_sweep_gxg.cuh"
#include "krcv_sort.cuh"
#include "krcv_prefix.cuh"
#include "krcv_window.cuh"
#include "krcv_ci.cuh"
#include "krcv_dense.cuh"
#include "krcv_kde.cuh"
#include "krcv_ll.cuh"
#include "krcv_hist.cuh"

namespace krcv {

// ---------------------------------------------------------------------------
// a1: pack + device-side validation
// ---------------------------------------------------------------------------
__global__ void pack_kernel(const double *__restrict__ x, const double *__restrict__ y, int n,
                            const double *__restrict__ h, int m,
                            uint64_t *__restrict__ keys, uint32_t *__restrict__ vals,
                            unsigned *__restrict__ status)
{
    const int stride = gridDim.x * blockDim.x;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned bad = 0, gbad = 0;
    for (int i = tid; i < n; i += stride) {
        double xv = x[i], yv = y[i];
        bad += (!isfinite(xv) || !isfinite(yv)) ? 1u : 0u;
        keys[i] = order_key(xv);
        vals[i] = static_cast<uint32_t>(i);
    }
    for (int b = tid; b < m; b += stride) {
        double hb = h[b];
        gbad += (!isfinite(hb) || !(hb > 0.0) || (b > 0 && hb < h[b - 1])) ? 1u : 0u;
    }
    if (bad) atomicAdd(&status[1], bad);
    if (gbad) atomicAdd(&status[0], gbad);
}

// a2 (second half): gather (x, y) into sorted order as one 16-byte record,
// with kPad (-inf, 0) / (+inf, 0) sentinels before and after (xy points at
// the first real record).  Also resets the sweep's tile counter.
__global__ void gather_kernel(const double *__restrict__ x, const double *__restrict__ y,
                              const uint32_t *__restrict__ order, int n, double2 *__restrict__ xy,
                              uint32_t *__restrict__ perm, int *__restrict__ tile_counter)
{
    pdl_wait();  // krcv_pdl.cuh
    const int stride = gridDim.x * blockDim.x;
    const int tid = blockIdx.x * blockDim.x + threadIdx.x;
    for (int k = tid; k < n; k += stride) {
        uint32_t i = order[k];
        xy[k] = make_double2(x[i], y[i]);
        perm[k] = i;
    }
    if (tid < kPad) {
        xy[-1 - tid] = make_double2(-INFINITY, 0.0);
        xy[n + tid] = make_double2(INFINITY, 0.0);
    }
    if (tid == 0) *tile_counter = 0;
}

// ---------------------------------------------------------------------------
// a3 + a4: the sweep -- see krcv_sweep.cuh
// ---------------------------------------------------------------------------
// ---------------------------------------------------------------------------
// finalize: CV = S/n, arg-min (Q11), status.  One CTA of THREADS threads;
// the paper's min-reduction kernel (P@24653).  Reads the partial vector with
// ld.global.cg (it may have been written by other CTAs of the same launch).
// ---------------------------------------------------------------------------
template <int THREADS>
__device__ __forceinline__ void finalize_body(const double *partial, long long n, int m, double *__restrict__ cv,
                                              long long *__restrict__ neff, int *__restrict__ best,
                                              int *__restrict__ status, double *sv, int *si)
{
    double bv = 0.0;
    int bi = -1;
    for (int b = threadIdx.x; b < m; b += THREADS) {
        const double v = __ldcg(partial + b) / (double)n;
        cv[b] = v;
        if (neff) neff[b] = (long long)__ldcg(partial + m + b);
        if (!isnan(v) && (bi < 0 || v < bv)) {  // strided order: b ascending per thread
            bv = v;
            bi = b;
        }
    }
    // (min value, lowest index) is associative and commutative: any tree
    // gives the same index.  Butterfly per warp, then warp 0 over the warps.
    auto take = [](double &mv, int &mi, double ov, int oi) {
        if (oi >= 0 && (mi < 0 || ov < mv || (ov == mv && oi < mi))) {
            mv = ov;
            mi = oi;
        }
    };
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
        take(bv, bi, __shfl_xor_sync(0xffffffffu, bv, o), __shfl_xor_sync(0xffffffffu, bi, o));
    if ((threadIdx.x & 31) == 0) {
        sv[threadIdx.x >> 5] = bv;
        si[threadIdx.x >> 5] = bi;
    }
    __syncthreads();
    if (threadIdx.x < 32) {
        bv = threadIdx.x < THREADS / 32 ? sv[threadIdx.x] : 0.0;
        bi = threadIdx.x < THREADS / 32 ? si[threadIdx.x] : -1;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
            take(bv, bi, __shfl_xor_sync(0xffffffffu, bv, o), __shfl_xor_sync(0xffffffffu, bi, o));
    }
    if (threadIdx.x == 0) {
        *best = bi < 0 ? 0 : bi;
        int st = KR_OK;
        if (__ldcg(partial + 2 * m) != 0.0) st = KR_EGRID;
        else if (__ldcg(partial + 2 * m + 1) != 0.0) st = KR_ENONFINITE;
        *status = st;
    }
}

constexpr int kFinThreads = 1024;

__global__ void __launch_bounds__(kFinThreads)
finalize_kernel(const double *__restrict__ partial, long long n, int m, double *__restrict__ cv,
                long long *__restrict__ neff, int *__restrict__ best, int *__restrict__ status)
{
    __shared__ double sv[kFinThreads];
    __shared__ int si[kFinThreads];
    finalize_body<kFinThreads>(partial, n, m, cv, neff, best, status, sv, si);
}

// ---------------------------------------------------------------------------
// a5: fixed-order column reduction of the tile partials (the paper's
// "summation reduction ... performed k times", P@23970, as one launch).
// With fin != nullptr (single-GPU whole search, kr_cv_grid_async) the last
// CTA to finish also runs the finalize (threadfence + completion counter),
// saving a launch; the counter is reset for the next call.
// ---------------------------------------------------------------------------
constexpr int kReduceThreads = 256;

struct FinOut {
    long long n;
    double *cv;
    long long *neff;
    int *best, *status;
    unsigned *done;
};

// Partial layouts: [m][ntiles] with every column entry valid (slots == 0:
// one partial per 32-row tile, uint8 counts), or win_kernel's warp slots
// (slots = S > 0, uint32 counts, krcv_window.cuh): bandwidth b of chunk
// c = b / bc was run by all S slots when ntiles >= S, else by the ntiles slots
// (c ntiles + t) mod S, t = 0 .. ntiles-1 -- summed in that (fixed) order.
template <typename CountT>
__global__ void __launch_bounds__(kReduceThreads)
reduce_kernel(const double *__restrict__ tileS, const CountT *__restrict__ tileN, int ntiles, int m,
              const unsigned *__restrict__ status, double *__restrict__ partial, FinOut fin, int slots, int bc)
{
    pdl_wait();  // krcv_pdl.cuh
    __shared__ double sS[kReduceThreads];
    __shared__ long long sN[kReduceThreads];
    __shared__ int sI[kReduceThreads];
    __shared__ bool last;
    for (int b = blockIdx.x; b < m; b += gridDim.x) {
        double a = 0.0;
        long long cnt = 0;
        if (slots == 0) {
            const double *col = tileS + (size_t)b * ntiles;
            const CountT *ncol = tileN + (size_t)b * ntiles;
            for (int t = threadIdx.x; t < ntiles; t += kReduceThreads) {
                a += col[t];
                cnt += ncol[t];
            }
        } else {
            const int nsl = ntiles >= slots ? slots : ntiles;
            const int first = ntiles >= slots ? 0 : (int)(((int64_t)(b / bc) * ntiles) % slots);
            const double *col = tileS + (size_t)b * slots;
            const CountT *ncol = tileN + (size_t)b * slots;
            for (int q = threadIdx.x; q < nsl; q += kReduceThreads) {
                int sl = first + q;
                sl = sl >= slots ? sl - slots : sl;
                a += col[sl];
                cnt += ncol[sl];
            }
        }
        // fixed tree: butterfly within each warp, then warp 0 adds the eight
        // warp sums in order (bit-reproducible, one barrier)
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            a += __shfl_xor_sync(0xffffffffu, a, o);
            cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
        }
        const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
        if (lane == 0) {
            sS[w] = a;
            sN[w] = cnt;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            double t = 0.0;
            long long c = 0;
#pragma unroll
            for (int q = 0; q < kReduceThreads / 32; q++) {
                t += sS[q];
                c += sN[q];
            }
            partial[b] = t;
            partial[m + b] = (double)c;
        }
        __syncthreads();
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        partial[2 * m] = (double)status[0];
        partial[2 * m + 1] = (double)status[1];
    }
    if (fin.cv == nullptr) return;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) last = atomicAdd(fin.done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!last) return;
    __threadfence();
    finalize_body<kReduceThreads>(partial, fin.n, m, fin.cv, fin.neff, fin.best, fin.status, sS, sI);
    if (threadIdx.x == 0) *fin.done = 0u;
}

// ---------------------------------------------------------------------------
// Programmatic dependent launch (krcv_pdl.cuh): only kernels that start with
// pdl_wait() are launched this way.  KRCV_PDL=0 launches them plainly.
// ---------------------------------------------------------------------------
static bool pdl_enabled()
{
    static const bool v = [] {
        const char *e = getenv("KRCV_PDL");
        return !(e && e[0] == '0');
    }();
    return v;
}

template <typename... KArgs, typename... Args>
static void launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                       Args... args)
{
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);  // errors surface via cudaGetLastError
}

// ---------------------------------------------------------------------------
// Per-device launch facts, safe under concurrent first calls (include/krcv.h
// promises re-entrant entry points): the SM count of each device, and the
// resident CTAs per SM of each (kernel, block size, smem) on each device,
// computed once under a mutex and cached.  Environment overrides are read
// into function-local statics with thread-safe (C++11 "magic static")
// initialisation.
// ---------------------------------------------------------------------------
struct DevInfo {
    int sms = 148;
};

static int current_device()
{
    int dev = 0;
    cudaGetDevice(&dev);
    return dev;
}

static const DevInfo &dev_info()
{
    constexpr int kMaxDev = 64;
    static std::mutex mu;
    static DevInfo info[kMaxDev];
    static bool have[kMaxDev] = {};
    const int dev = current_device();
    const int d = dev >= 0 && dev < kMaxDev ? dev : 0;
    std::lock_guard<std::mutex> g(mu);
    if (!have[d]) {
        int sms = 0;
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess && sms > 0)
            info[d].sms = sms;
        else
            cudaGetLastError();
        have[d] = true;
    }
    return info[d];
}

// partial slots win_kernel may use on this device (workspace sizing): at
// most 64 resident warps per SM (the uniform instantiation's 56 registers
// allow 9 CTAs = 36 warps per SM)
static int64_t win2_max_slots() { return (int64_t)dev_info().sms * 64; }

static int occupancy(const void *func, int threads, size_t smem = 0)
{
    struct Key {
        int dev;
        const void *f;
        int threads;
        size_t smem;
        int value;
    };
    static std::mutex mu;
    static std::vector<Key> cache;
    const int dev = current_device();
    std::lock_guard<std::mutex> g(mu);
    for (const Key &k : cache)
        if (k.dev == dev && k.f == func && k.threads == threads && k.smem == smem) return k.value;
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, func, threads, smem) != cudaSuccess) {
        cudaGetLastError();
        b = 1;
    }
    if (b < 1) b = 1;
    cache.push_back(Key{dev, func, threads, smem, b});
    return b;
}

// ---------------------------------------------------------------------------
// tracing and fault injection (krcv_internal.h)
// ---------------------------------------------------------------------------
NvtxScope::NvtxScope(const char *name) { nvtxRangePushA(name); }
NvtxScope::~NvtxScope() { nvtxRangePop(); }

bool injected_failure(const char *stage)
{
    const char *e = getenv("KRCV_FAIL_AT");
    if (!e || strcmp(e, stage) != 0) return false;
    char buf[96];
    snprintf(buf, sizeof buf, "injected failure at %s (KRCV_FAIL_AT)", stage);
    set_error_text(buf);
    return true;
}

// ---------------------------------------------------------------------------
// host-side launch helpers
// ---------------------------------------------------------------------------
// CUB onesweep falls back to a single-tile kernel below this many keys
// (policy-dependent; verified from the ncu launch list).
constexpr int64_t kCubSingleTile = 0;

static inline size_t align256(size_t v) { return (v + 255) & ~size_t(255); }

// Workspace classes (size the partials per algorithm; the KDE
// sum-B block only for the KDE entry points).  Everything before the bucket
// table has the same offset in every class (kr_cv_refine reuses it in place).
int ws_class_for(int32_t algo, int32_t kernel, int64_t rows)
{
    if (algo == KR_ALGO_AUTO) algo = kernel == KR_GAUSSIAN ? KR_ALGO_DENSE : auto_algo(rows, rows, 0, kernel);
    return algo == KR_ALGO_SWEEP ? kWsSweep : kWsDefault;
}

bool ws_layout(int64_t n, int32_t m, WsLayout *L, int cls)
{
    size_t cub_bytes = 0, cub32 = 0;
    cudaError_t e = cub::DeviceRadixSort::SortPairs(
        nullptr, cub_bytes, (const uint64_t *)nullptr, (uint64_t *)nullptr,
        (const uint32_t *)nullptr, (uint32_t *)nullptr, (int)n, 0, 64, (cudaStream_t)0);
    if (e == cudaSuccess)
        e = cub::DeviceRadixSort::SortPairs(nullptr, cub32, (const uint32_t *)nullptr, (uint32_t *)nullptr,
                                            (const uint32_t *)nullptr, (uint32_t *)nullptr, (int)n, 0, 32,
                                            (cudaStream_t)0);
    if (e != cudaSuccess) {
        set_cuda_error("cub::DeviceRadixSort::SortPairs(size query)", (int)e);
        return false;
    }
    cub_bytes = cub_bytes > cub32 ? cub_bytes : cub32;
    const int64_t ntiles = max_tiles(n);
    size_t off = 0;
    const size_t npad = (size_t)((n + kChunk - 1) / kChunk) * kChunk;  // chunked rank sort
    L->keys_in = off;  off = align256(off + sizeof(uint64_t) * npad);
    L->keys_out = off; off = align256(off + sizeof(uint64_t) * npad);
    L->vals_in = off;  off = align256(off + sizeof(uint32_t) * npad);
    L->vals_out = off; off = align256(off + sizeof(uint32_t) * npad);
    L->xy = off;       off = align256(off + sizeof(double2) * ((size_t)n + 2 * kPad));
    L->counter = off;  off = align256(off + sizeof(int) * 32);  // tile counter
    L->perm = off;     off = align256(off + sizeof(uint32_t) * (size_t)n);
    // window-prefix path (krcv_prefix.cuh)
    const size_t nch = (size_t)((n + kPfxTileMin) / kPfxTileMin);  // most tiles covering P[0..n]
    L->pstride = (int64_t)(((size_t)n + 1 + 15) & ~size_t(15));
    L->nch = (int64_t)nch;
    L->xs = off;       off = align256(off + sizeof(double) * ((size_t)n + 2 * kPad));
    // prefix moments: SoA planes (KDE, local-linear: 8 x 2 x pstride doubles) or the
    // blocked records of the NW sets (2 x 5 x pk_slots doubles at most)
    const size_t pfx_soa = sizeof(double2) * kPfxMoments * (size_t)L->pstride;
    const size_t pfx_rec = sizeof(double) * 2 * pk_lo_off<KR_EPANECHNIKOV>((int)L->pstride);
    L->pfx = off;      off = align256(off + (pfx_soa > pfx_rec ? pfx_soa : pfx_rec));
    L->ptot = off;     off = align256(off + sizeof(double2) * kPfxMoments * nch);
    // anchored hi records of the Epanechnikov fast path (krcv_window.cuh), window-prefix classes
    L->pfxa = off;
    if (cls == kWsDefault || cls == kWsAll)  // anchors_for: 0 below n = 50,000 and above kAncMaxN
        off = align256(off + sizeof(double) * anchors_for(n) * pk_lo_off<KR_EPANECHNIKOV>((int)L->pstride));
    // 256 B: counters, max|y|, density statistic (bytes 0-31), BktParams (32), q32 key range (64-79)
    L->status = off;   off = align256(off + 8 * sizeof(unsigned));
    L->cub = off;      off = align256(off + cub_bytes);
    // m-dependent buffers last: everything above has the same offset for any
    // m, so a refinement level with another grid size can reuse the sorted
    // arrays and prefix moments in place (kr_cv_refine)
    // bucket table of win_kernel (krcv_window.cuh): int32 [Qmax + 1], Qmax = min(kBktFmax n, kBktQmax)
    const int64_t qmax = (int64_t)kBktFmax * n < kBktQmax ? (int64_t)kBktFmax * n : kBktQmax;
    L->bt = off;       off = align256(off + sizeof(int) * (size_t)(qmax + 1));
    // partials: one per win_kernel warp slot (uint32 counts), one per 32-row
    // tile (r01 window, local-linear, histogram, dense, KDE; uint8 counts) and,
    // for the sweep class, one per 32/G-row tile of the split sweep
    const size_t slots = (size_t)win2_max_slots();
    const size_t t32 = (size_t)((n + 31) / 32);
    size_t tiles = t32;
    if (cls == kWsSweep || cls == kWsAll) tiles = (size_t)ntiles > tiles ? (size_t)ntiles : tiles;
    L->tileS = off;    off = align256(off + sizeof(double) * (tiles > slots ? tiles : slots) * (size_t)m);
    const size_t nbytes = tiles > 4 * slots ? tiles : 4 * slots;
    L->tileN = off;    off = align256(off + nbytes * (size_t)m);
    L->tileB = off;
    if (cls == kWsKde || cls == kWsAll) off = align256(off + sizeof(double) * t32 * (size_t)m);  // KDE sum B
    L->partial = off;  off = align256(off + sizeof(double) * (size_t)KR_PARTIAL_LEN(m));
    L->cub_bytes = cub_bytes;
    L->total = off;
    L->ntiles_max = ntiles;
    return true;
}

// Lanes per row group.  Measured on B200 (profiles/): G = 4
// is fastest for both sweep variants on C2-C5 (G = 1/2 leave the FP64 pipe
// idle at 1-2 warps per scheduler on small shards; G = 8 adds epilogue and
// combine overhead).  KRCV_SWEEP_G overrides (1, 2, 4; 8 for split).
int sweep_G(int64_t /*rows*/)
{
    static const int forced = [] {
        const char *e = getenv("KRCV_SWEEP_G");
        const int g = e ? atoi(e) : 0;
        return (g == 1 || g == 2 || g == 4 || g == 8) ? g : 0;
    }();
    return forced ? forced : 4;
}

static int64_t tiles_for(int64_t rows, int G) { return (rows * G + 31) / 32; }

// Upper bound of tile slots for any shard of n rows and either variant:
// split uses 32/G rows per tile, gxg 32.
int64_t max_tiles(int64_t n) { return tiles_for(n, sweep_G(n)); }

static bool getenv_flag(const char *name)
{
    const char *e = getenv(name);
    return e && e[0] && e[0] != '0';
}

static int grid_for(int64_t work, int threads)
{
    int64_t b = (work + threads - 1) / threads;
    if (b < 1) b = 1;
    if (b > 148 * 16) b = 148 * 16;
    return (int)b;
}

// Sweep variant for a shard of `rows` rows: 0 = split (G lanes per row),
// 1 = gxg (G lanes x G adjacent rows with shared moments).  gxg halves the
// C4 sweep (1e6 rows) but degrades on heavy-tailed data with few rows per
// unit of x (C5) and on small shards (C2); measured crossover ~4e5 rows
// (DESIGN.md §6).  KRCV_SWEEP=split|gxg overrides.
int sweep_variant(int64_t rows)
{
    static const int v = [] {
        const char *e = getenv("KRCV_SWEEP");
        return !e ? 2 : (e[0] == 's' ? 0 : (e[0] == 'g' ? 1 : 2));
    }();
    if (v != 2) return v;
    return rows >= kGxgRows ? 1 : 0;
}

template <int KERN, int G, bool GXG>
static void launch_sweep_g(const double2 *xy, int n, const double *h, int m, int lo, int hi, int ntiles,
                           double *tileS, uint8_t *tileN, int *counter, cudaStream_t st)
{
    // CTAs per SM at full occupancy (persistent grid)
    const int resident = occupancy(GXG ? (const void *)sweep_gxg_kernel<KERN, G> : (const void *)sweep_kernel<KERN, G>,
                                   kSweepThreads);
    const int sms = dev_info().sms;
    int blocks = (ntiles + kSweepWarps - 1) / kSweepWarps;
    if (blocks > sms * resident) blocks = sms * resident;
    if (GXG)
        sweep_gxg_kernel<KERN, G><<<blocks, kSweepThreads, 0, st>>>(xy, n, h, m, lo, hi, ntiles, tileS, tileN,
                                                                    counter);
    else
        sweep_kernel<KERN, G><<<blocks, kSweepThreads, 0, st>>>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter);
}

template <int KERN>
static void launch_sweep(int G, const double2 *xy, int n, const double *h, int m, int lo, int hi, int ntiles,
                         double *tileS, uint8_t *tileN, int *counter, cudaStream_t st)
{
    if (sweep_variant(hi - lo) == 1) {
        switch (G) {
        case 1: launch_sweep_g<KERN, 1, true>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
        case 2: launch_sweep_g<KERN, 2, true>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
        default: launch_sweep_g<KERN, 4, true>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
        }
        return;
    }
    switch (G) {
    case 1: launch_sweep_g<KERN, 1, false>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
    case 2: launch_sweep_g<KERN, 2, false>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
    case 4: launch_sweep_g<KERN, 4, false>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
    default: launch_sweep_g<KERN, 8, false>(xy, n, h, m, lo, hi, ntiles, tileS, tileN, counter, st); break;
    }
}

// Optional stage timing (kr_profile_enable / kr_profile_read), thread-local.
// Events: 0 start, 1 after pack+sort+gather, 2 after the prefix build (equal
// to 1 on the sweep path), 3 after the sweep / window kernel, 4 after reduce.
constexpr int kProfEvents = 5;
struct Prof {
    bool on = false;
    bool recorded = false;
    cudaEvent_t ev[kProfEvents] = {nullptr, nullptr, nullptr, nullptr, nullptr};
    int64_t launches = 0;
    int algo = 0;
};
static thread_local Prof g_prof;

bool prof_enabled() { return g_prof.on; }

static void prof_mark(int k, cudaStream_t st)
{
    if (!g_prof.on) return;
    if (!g_prof.ev[k]) cudaEventCreate(&g_prof.ev[k]);
    // inside a stream capture (GridSearch(graph=True)) the record must be an
    // external event-record node so that every graph replay records it
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(st, &cs);
    if (cs == cudaStreamCaptureStatusActive)
        cudaEventRecordWithFlags(g_prof.ev[k], st, cudaEventRecordExternal);
    else
        cudaEventRecord(g_prof.ev[k], st);
}

// Kernel launches CUB's radix sort makes for `n` 64-bit keys.  Onesweep:
// one histogram kernel + one exclusive-scan kernel + one pass per 8-bit
// digit; below the single-tile threshold a single kernel.  (Cross-checked
// against the ncu launch list, profiles/.)
static int64_t cub_sort_launches(int64_t n) { return n <= kCubSingleTile ? 1 : 2 + 64 / 8; }

// Small-n sort chunk configuration: 0 = 256x4 (1024), 1 = 256x8 (2048),
// 2 = 512x8 (4096), 3 = 256x2 (512), 4 = 128x2 (256) records per CTA.
// Measured (profiles/r01v_*, r01al_*): 1024 beats 2048 / 4096 at C2 and C3;
// 512 beats 1024 at C2 (sort 26 -> 22 us) -- smaller chunks sort faster on
// more SMs while the extra chunk pairs of the rank step stay cheap at small
// n.  KRCV_CHUNK=0..4 overrides.
int chunk_config(int64_t n)
{
    static const int forced = [] {
        const char *e = getenv("KRCV_CHUNK");
        return (e && e[0] >= '0' && e[0] <= '4') ? e[0] - '0' : 5;
    }();
    if (forced != 5) return forced;
    return n <= 40000 ? 3 : 0;
}

template <int T, int I>
static void launch_rank_sort(const double *d_x, const double *d_y, int n, const double *d_h, int m, uint64_t *keys,
                             uint32_t *khi, uint32_t *idx, int *rank, unsigned *status, int nchunks, cudaStream_t st)
{
    chunk_sort_kernel<T, I><<<nchunks, T, 0, st>>>(d_x, d_y, n, d_h, m, keys, khi, idx, rank, status);
    if (nchunks <= 1) return;
    launch_pdl(rank_count_kernel<T, I>, dim3(nchunks, nchunks), dim3(T), 0, st, keys, khi, idx, rank);
}

// KR_ALGO_AUTO: the window-prefix path does O(n m log) work against the
// sweep's O(n^2); measured faster on every BASELINE config.
// KRCV_ALGO=sweep|prefix overrides (benchmarks, A/B tests).
int auto_algo(int64_t /*n*/, int64_t /*rows*/, int32_t /*m*/, int32_t /*kernel*/)
{
    static const int forced = [] {
        const char *e = getenv("KRCV_ALGO");
        return !e ? 0 : (e[0] == 's' ? KR_ALGO_SWEEP : (e[0] == 'p' ? KR_ALGO_PREFIX : (e[0] == 'h' ? KR_ALGO_HIST : 0)));
    }();
    return forced ? forced : KR_ALGO_PREFIX;
}

// Records per thread of the prefix build: 1 (256-record tiles, more CTAs)
// up to 2^18 records, 4 above.  KRCV_PFX_ITEMS=1|4 overrides.
// 0 = the one-CTA build (pfx_one_cta_kernel) for n <= kPfxOneCtaMax: its
// per-thread sequential dd chains only pay off for a few records per thread
// (profiles/experiments/r01be_*).
// KRCV_PFX_ITEMS=0|1|4 overrides.
constexpr int kPfxOneCtaMax = 1024;  // measured: C1 (n = 1,000) 10.2 -> 8.2 us, C2 (n = 20,000) 18 -> 187 us

// KRCV_PFX_ITEMS=0|1|4 forces the build's tile size (A/B runs), else -2
static int pfx_items_forced()
{
    static const int forced = [] {
        const char *e = getenv("KRCV_PFX_ITEMS");
        const int v = e ? atoi(e) : -2;
        return (v == 0 || v == 1 || v == 4) ? v : -2;
    }();
    return forced;
}

// The moment sets without the fused build (KDE, local-linear): one CTA for
// n <= 1,024, then 256-record tiles, 1,024-record tiles from n > 131,072
// (measured, profiles/r02/r02ag_*: C5 build 55 -> 51 us, equal at C3).  The
// regression sets take the fused build wherever its tiles are co-resident,
// at n <= 1,024 too (C1 build 14.3 -> 12.3 us, step 0.039 -> 0.035 ms,
// profiles/r02/r02ak_*).
static int pfx_items(int n)
{
    const int forced = pfx_items_forced();
    if (forced != -2) return forced;
    return n <= kPfxOneCtaMax ? 0 : (n <= (1 << 17) ? 1 : kPfxItemsMax);
}

static void launch_bkt_fill(int n, const WsLayout &L, char *ws, cudaStream_t st);

// win_kernel's anchored records (Epanechnikov, after the prefix build): one
// thread per (index 0..n, anchor), only the copies of the anchors whose
// regions hold rows [row_lo, row_hi) of this call (a shard of P ranks builds
// about J / P of them).
template <int KERN>
static int launch_anchors(int n, const WsLayout &L, char *ws, cudaStream_t st, bool table, int row_lo, int row_hi)
{
    const int J = anchors_for(n);
    if (KERN != KR_EPANECHNIKOV || !table || J == 0 || row_hi <= row_lo) return 0;
    const int j0 = anc_of(row_lo, J, n), j1 = anc_of(row_hi - 1, J, n);
    const double *xs = reinterpret_cast<const double *>(ws + L.xs) + kPad;
    const double *P = reinterpret_cast<const double *>(ws + L.pfx);
    double *PA = reinterpret_cast<double *>(ws + L.pfxa);
    double *OJ = reinterpret_cast<double *>(ws + L.status + 96);
    const int64_t blocks = ((int64_t)n + kAncThreads) / kAncThreads * (j1 - j0 + 1);  // indices 0..n per copy
    launch_pdl(anchor_kernel<KR_EPANECHNIKOV>, dim3((unsigned)blocks), dim3(kAncThreads), 0, st, xs, P,
               (int)L.pstride, n, J, j0, j1 - j0 + 1, PA, OJ);
    return 1;
}

// The O(n) build of the window-prefix path: prefix moments, xs and (table:
// win_kernel's) the bucket table.  Returns the launches enqueued.
template <int KERN>
static int launch_prefix_build(const double2 *xy, int n, const WsLayout &L, char *ws, cudaStream_t st,
                               bool table = false, int row_lo = 0, int row_hi = 0)
{
    double *xs = reinterpret_cast<double *>(ws + L.xs) + kPad;
    double *P = reinterpret_cast<double *>(ws + L.pfx);
    double2 *tot = reinterpret_cast<double2 *>(ws + L.ptot);
    unsigned long long *ymax = reinterpret_cast<unsigned long long *>(ws + L.status + 4 * sizeof(unsigned));
    unsigned long long *gap = reinterpret_cast<unsigned long long *>(ws + L.status + 6 * sizeof(unsigned));
    const int items = pfx_items(n);
    const int tiles1 = (n + kPfxThreads) / kPfxThreads;  // 256-record tiles covering P[0..n]
    const bool fusable = items == 1 || (items == 0 && pfx_items_forced() == -2);
    if (fusable && PfxRec<KERN>::S && tiles1 <= dev_info().sms && !getenv_flag("KRCV_PFX_UNFUSED")) {
        // every tile co-resident (<= one CTA per SM): the fused build
        unsigned *arrive = reinterpret_cast<unsigned *>(ws + L.status) + 3;  // zeroed by the status memset
        int *BT = table ? reinterpret_cast<int *>(ws + L.bt) : nullptr;
        BktParams *prm = reinterpret_cast<BktParams *>(ws + L.status + 32);
        launch_pdl(pfx_fused_kernel<KERN>, dim3(tiles1), dim3(kFusedPfxThreads), 0, st, xy, n, tot, tiles1, ymax,
                   gap, P, (int)L.pstride, xs, BT, prm, arrive);
        return 1 + launch_anchors<KERN>(n, L, ws, st, table, row_lo, row_hi);
    }
    int launches = 2;
    if (items == 0) {
        pfx_one_cta_kernel<KERN><<<1, kPfx1Threads, 0, st>>>(xy, n, P, (int)L.pstride, xs, ymax, gap);
        launches = 1;
    } else if (items == 1) {
        const int ntiles = (n + kPfxThreads) / kPfxThreads;  // tiles covering P[0..n]
        launch_pdl(pfx_tile_reduce_kernel<KERN, 1>, dim3(ntiles), dim3(kPfxThreads), 0, st, xy, n, tot, ntiles, ymax);
        launch_pdl(pfx_tile_scan_kernel<KERN, 1>, dim3(ntiles), dim3(kPfxThreads), 0, st, xy, n,
                   (const double2 *)tot, ntiles, P, (int)L.pstride, xs, gap);
    } else {
        const int ntiles = (n + kPfxThreads * kPfxItemsMax) / (kPfxThreads * kPfxItemsMax);
        launch_pdl(pfx_tile_reduce_kernel<KERN, kPfxItemsMax>, dim3(ntiles), dim3(kPfxThreads), 0, st, xy, n, tot,
                   ntiles, ymax);
        launch_pdl(pfx_tile_scan_kernel<KERN, kPfxItemsMax>, dim3(ntiles), dim3(kPfxThreads), 0, st, xy, n,
                   (const double2 *)tot, ntiles, P, (int)L.pstride, xs, gap);
    }
    if (table) {
        launch_bkt_fill(n, L, ws, st);
        launches += 1;
    }
    return launches + launch_anchors<KERN>(n, L, ws, st, table, row_lo, row_hi);
}

// Window kernel of r01 (window_kernel<K> / window_kernel_b2), kept for A/B
// runs: K consecutive rows per lane (K = 1, 2) or one row per lane with two
// bandwidths per step (3).  KRCV_WIN_K overrides.
int win_rows_per_lane(int64_t rows)
{
    static const int forced = [] {
        const char *e = getenv("KRCV_WIN_K");
        const int k = e ? atoi(e) : 0;
        return (k >= 1 && k <= 3) ? k : 0;
    }();
    if (forced) return forced;
    // measured (profiles/r01t_*, r01u_*, r01af_*): two consecutive rows per
    // lane up to 5e4 rows, above one row per lane with two bandwidths per step
    return rows <= 50000 ? 2 : 3;
}

static int win_lane_rows(int K) { return K == 3 ? 1 : K; }

template <int KERN, int K>
static void launch_window_k(const double2 *xy, int n, const double *h, int m, int lo, int hi, int ntiles,
                            const WsLayout &L, char *ws, double *tileS, uint8_t *tileN, int *counter,
                            cudaStream_t st)
{
    const DevInfo &di = dev_info();
    const int resident = occupancy(K == 3 ? (const void *)window_kernel_b2<KERN> : (const void *)window_kernel<KERN, K == 3 ? 1 : K>,
                                   kWinThreads);
    // Split the bandwidth loop into nbc chunks until there are enough warp
    // tasks to fill every SM (~kWinTasksPerSM resident warps each), keeping
    // >= kWinMinBper bandwidths per chunk to amortise the cold searches.
    const int64_t want = (int64_t)di.sms * kWinTasksPerSM;
    int nbc = (int)((want + ntiles - 1) / ntiles);
    nbc = nbc < 1 ? 1 : nbc;
    const int max_nbc = (m + kWinMinBper - 1) / kWinMinBper;
    if (nbc > max_nbc) nbc = max_nbc;
    if (nbc < 1) nbc = 1;
    const int64_t tasks = (int64_t)ntiles * nbc;
    int blocks = (int)((tasks + kWinWarps - 1) / kWinWarps);
    if (blocks > di.sms * resident) blocks = di.sms * resident;
    const double *xs = reinterpret_cast<const double *>(ws + L.xs) + kPad;
    const double *P = reinterpret_cast<const double *>(ws + L.pfx);
    const unsigned long long *ymax =
        reinterpret_cast<const unsigned long long *>(ws + L.status + 4 * sizeof(unsigned));
    if (K == 3)
        launch_pdl(window_kernel_b2<KERN>, dim3(blocks), dim3(kWinThreads), 0, st, xs, (const double2 *)xy, P,
                   (int)L.pstride, h, m, n, lo, hi, ntiles, nbc, ymax, tileS, tileN, counter);
    else
        launch_pdl(window_kernel<KERN, K == 3 ? 1 : K>, dim3(blocks), dim3(kWinThreads), 0, st, xs,
                   (const double2 *)xy, P, (int)L.pstride, h, m, n, lo, hi, ntiles, nbc, ymax, tileS, tileN,
                   counter);
}

template <int KERN>
static void launch_window(int K, const double2 *xy, int n, const double *h, int m, int lo, int hi, int ntiles,
                          const WsLayout &L, char *ws, double *tileS, uint8_t *tileN, int *counter,
                          cudaStream_t st)
{
    switch (K) {
    case 1: launch_window_k<KERN, 1>(xy, n, h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st); break;
    case 3: launch_window_k<KERN, 3>(xy, n, h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st); break;
    default: launch_window_k<KERN, 2>(xy, n, h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st); break;
    }
}

// Window kernel selection: 1 = win_kernel (bucket-table lookups,
// krcv_window.cuh; default), 0 = r01's window_kernel / window_kernel_b2
// (KRCV_WIN=r01, A/B runs).
static bool use_win2()
{
    static const bool v = [] {
        const char *e = getenv("KRCV_WIN");
        return !(e && strcmp(e, "r01") == 0);
    }();
    return v;
}

// Task shape of win_kernel for a shard of `rows` rows: BC bandwidths per
// chunk (1 .. kWin2Chunk), so that there are about kWin2TasksPerWarp tasks per
// warp slot; S = the persistent grid's warp slots.
struct Win2Shape {
    int BC, nbc, ntiles, blocks, S;
};
// Task shape (measured, profiles/r02/r02v_*): about 16 tasks per warp slot
// (C3 1.192 -> 1.160 ms, C5 1.653 -> 1.600 ms against 8), but chunks of at
// least 3 bandwidths (C2: 16 per slot would mean one-bandwidth tasks, whose
// per-task row setup costs more than the balance gains: 65.5 -> 60.4 us
// window at 3 bandwidths).  A rule minimising the slot imbalance
// ceil(tasks / S) (BC + c0) instead (C2: 14-bandwidth chunks, one task per
// slot) measured slower at C2 / C3 / C5 (59 -> 70 us, +3 %, +5 %) and 1 %
// faster at C4: the chunk-major round-robin keeps few chunks -- a narrow
// band of bandwidths, so of boundary positions -- in flight, and large
// chunks widen it (profiles/r02/r02aj_*).
constexpr int kWin2TasksPerWarp = 16;
constexpr int kWin2MinChunk = 3;

template <int KERN>
static Win2Shape win2_shape(int64_t rows, int m)
{
    Win2Shape w;
    w.ntiles = (int)((rows + 31) / 32);
    // (both anchor variants have the same launch bounds: 64 registers, 8 CTAs per SM)
    const int resident = occupancy((const void *)win_kernel<KERN, false>, kWin2Threads);
    const int64_t slots = (int64_t)dev_info().sms * resident * kWin2Warps;
    static const int tpw = [] {  // KRCV_WIN2_TPW overrides (A/B runs)
        const char *e = getenv("KRCV_WIN2_TPW");
        const int v = e ? atoi(e) : 0;
        return v > 0 ? v : kWin2TasksPerWarp;
    }();
    static const int min_chunk = [] {  // KRCV_WIN2_MINCHUNK overrides (A/B runs)
        const char *e = getenv("KRCV_WIN2_MINCHUNK");
        const int v = e ? atoi(e) : 0;
        return v > 0 ? v : kWin2MinChunk;
    }();
    const int64_t target = (int64_t)tpw * slots;
    const int64_t npairs = (w.ntiles + kWin2Rows - 1) / kWin2Rows;
    int64_t bc = (int64_t)m * npairs / (target > 0 ? target : 1);
    bc = bc < min_chunk ? min_chunk : (bc > kWin2Chunk ? kWin2Chunk : bc);
    // too few tasks to fill the slots even at the minimum chunk (C1): smaller
    // chunks, up to one task per slot (C1 0.041 -> 0.037 ms, profiles/r02/r02aj_*)
    if (npairs * ((m + bc - 1) / bc) < slots) {
        const int64_t b = (m * npairs + slots - 1) / (slots > 0 ? slots : 1);
        bc = b < 1 ? 1 : (b < bc ? b : bc);
    }
    if (bc > m) bc = m;
    w.BC = (int)bc;
    w.nbc = (int)((m + bc - 1) / bc);
    // no more slots than tasks (a slot without a task would leave its partials unwritten)
    const int64_t tasks = (int64_t)((w.ntiles + kWin2Rows - 1) / kWin2Rows) * w.nbc;
    int64_t blocks = (int64_t)dev_info().sms * resident;
    if (blocks * kWin2Warps > win2_max_slots()) blocks = win2_max_slots() / kWin2Warps;
    if (blocks * kWin2Warps > tasks) blocks = tasks / kWin2Warps;
    if (blocks < 1) blocks = 1;
    w.blocks = (int)blocks;
    w.S = (int)blocks * kWin2Warps;
    return w;
}

// Anchors of the Epanechnikov fast path (krcv_window.cuh, anchor_kernel): J
// copies of the prefix hi words anchored at the centres of J index regions;
// 0 = none (the fast path reads the global records).  None below kAncMinN
// (C2: the window kernel gains nothing, the build costs 6 us); above, the
// most of 16 / 8 / 4 / 2 / 1 whose copies under one band of win_kernel's rows
// (its S slots x 64 rows in flight: J band / n + 1 copies of 40 n bytes) stay
// within kAncHotBytes of L2 -- measured C3 / C5 best at 8, C4 at 4
// (profiles/r02/r02aq_*).  KRCV_ANCHORS = 0 .. 8 overrides (A/B runs).
int anchors_for(int64_t n)
{
    static const int forced = [] {
        const char *e = getenv("KRCV_ANCHORS");
        return e ? atoi(e) : -1;
    }();
    if (n > kAncMaxN) return 0;
    if (forced >= 0) return forced > kAncMax ? kAncMax : forced;
    if (n < kAncMinN) return 0;
    const double band = (double)dev_info().sms * kWin2MinBlocks * kWin2Warps * 32.0 * kWin2Rows;  // rows in flight
    const double frac = band < (double)n ? band / (double)n : 1.0;
    for (int J = kAncMax; J > 1; J >>= 1) {
        const double hot = (J * frac + 1.0 < J ? J * frac + 1.0 : J) * 40.0 * (double)n;
        if (hot <= kAncHotBytes) return J;
    }
    return 1;
}

// the bucket table of win_kernel (krcv_window.cuh) from the sorted x: part of
// the O(n) build stage, after the prefix scan (which publishes the density
// statistic it sizes the table with)
static void launch_bkt_fill(int n, const WsLayout &L, char *ws, cudaStream_t st)
{
    const double *xs = reinterpret_cast<const double *>(ws + L.xs) + kPad;
    int *BT = reinterpret_cast<int *>(ws + L.bt);
    const unsigned long long *gap =
        reinterpret_cast<const unsigned long long *>(ws + L.status + 6 * sizeof(unsigned));
    BktParams *prm = reinterpret_cast<BktParams *>(ws + L.status + 32);
    const int64_t qmax = (int64_t)kBktFmax * n < kBktQmax ? (int64_t)kBktFmax * n : kBktQmax;
    int64_t blocks = (n + qmax + 1 + kBktTile - 1) / kBktTile;
    if (blocks > (int64_t)dev_info().sms * 8) blocks = (int64_t)dev_info().sms * 8;
    launch_pdl(bkt_fill_kernel, dim3((int)blocks), dim3(kBktFillThreads), 0, st, xs, n, gap, BT, prm);
}

template <int KERN>
static void launch_win2(const double2 *xy, int n, const double *h, int m, int lo, int hi, const Win2Shape &w,
                        const WsLayout &L, char *ws, double *tileS, uint32_t *tileN, cudaStream_t st)
{
    const double *xs = reinterpret_cast<const double *>(ws + L.xs) + kPad;
    const double *P = reinterpret_cast<const double *>(ws + L.pfx);
    int *BT = reinterpret_cast<int *>(ws + L.bt);
    const unsigned long long *ymax =
        reinterpret_cast<const unsigned long long *>(ws + L.status + 4 * sizeof(unsigned));
    const unsigned long long *gap =
        reinterpret_cast<const unsigned long long *>(ws + L.status + 6 * sizeof(unsigned));
    BktParams *prm = reinterpret_cast<BktParams *>(ws + L.status + 32);
    const double *PA = reinterpret_cast<const double *>(ws + L.pfxa);
    const double *OJ = reinterpret_cast<const double *>(ws + L.status + 96);
    Win2Sched sc;
    sc.npairs = (w.ntiles + kWin2Rows - 1) / kWin2Rows;
    sc.s_div = w.S / sc.npairs;
    sc.s_mod = w.S % sc.npairs;
    sc.ntasks = (long long)sc.npairs * w.nbc;
    const int J = KERN == KR_EPANECHNIKOV ? anchors_for(n) : 0;
    // the anchors launch_anchors built for these rows (the kernel clamps its choice to them)
    const int j0 = J > 0 && hi > lo ? anc_of(lo, J, n) : 0, j1 = J > 0 && hi > lo ? anc_of(hi - 1, J, n) : 0;
    if (J > 0)
        launch_pdl(win_kernel<KERN, KERN == KR_EPANECHNIKOV>, dim3(w.blocks), dim3(kWin2Threads), 0, st, xs, xy, P,
                   (int)L.pstride, (const int *)BT, (const BktParams *)prm, h, m, n, lo, hi, w.ntiles, w.BC, w.nbc,
                   ymax, tileS, tileN, PA, J, j0, j1, OJ, sc);
    else
        launch_pdl(win_kernel<KERN, false>, dim3(w.blocks), dim3(kWin2Threads), 0, st, xs, xy, P, (int)L.pstride,
                   (const int *)BT, (const BktParams *)prm, h, m, n, lo, hi, w.ntiles, w.BC, w.nbc, ymax, tileS,
                   tileN, PA, 0, 0, 0, OJ, sc);
}

// Histogram ordering (krcv_hist.cuh): `warps` warps per CTA (as many as the
// shared-memory histograms allow) share a 32-row tile; persistent CTAs.
template <int KERN>
static void launch_hist(int warps, const double *d_x, const double *d_y, const uint32_t *perm, const double2 *xy,
                        const double *h, int m, int n, int lo, int hi, int ntiles, double *tileS, uint8_t *tileN,
                        int *counter, cudaStream_t st)
{
    const size_t smem = hist_smem_bytes(m, warps);
    cudaFuncSetAttribute(hist_kernel<KERN>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const int resident = occupancy((const void *)hist_kernel<KERN>, warps * 32, smem);
    const int sms = dev_info().sms;
    int blocks = ntiles;  // one 32-row tile per CTA iteration
    if (blocks > sms * resident) blocks = sms * resident;
    hist_kernel<KERN><<<blocks, warps * 32, smem, st>>>(d_x, d_y, perm, xy, h, m, n, lo, hi, ntiles, tileS, tileN,
                                                         counter);
}

// Local-linear window kernel (krcv_ll.cuh): one row per lane, the same
// task split as window_kernel.
template <int KERN>
static void launch_ll_window(const double2 *xy, int n, const double *h, int m, int lo, int hi, int ntiles,
                             const WsLayout &L, char *ws, double *tileS, uint8_t *tileN, int *counter,
                             cudaStream_t st)
{
    const int resident = occupancy((const void *)ll_window_kernel<KERN>, kWinThreads);
    const int sms = dev_info().sms;
    const int64_t want = (int64_t)sms * kWinTasksPerSM;
    int nbc = (int)((want + ntiles - 1) / ntiles);
    const int max_nbc = (m + kWinMinBper - 1) / kWinMinBper;
    if (nbc > max_nbc) nbc = max_nbc;
    if (nbc < 1) nbc = 1;
    const int64_t tasks = (int64_t)ntiles * nbc;
    int blocks = (int)((tasks + kWinWarps - 1) / kWinWarps);
    if (blocks > sms * resident) blocks = sms * resident;
    const double *xs = reinterpret_cast<const double *>(ws + L.xs) + kPad;
    const double *P = reinterpret_cast<const double *>(ws + L.pfx);
    const unsigned long long *ymax =
        reinterpret_cast<const unsigned long long *>(ws + L.status + 4 * sizeof(unsigned));
    // KRCV_LL_STATS=1 (debug): count the branches taken, print to stderr
    unsigned long long *stats = nullptr;
    const bool want_stats = getenv_flag("KRCV_LL_STATS");
    if (want_stats && cudaMalloc(&stats, 4 * sizeof(unsigned long long)) != cudaSuccess) stats = nullptr;
    if (stats) cudaMemsetAsync(stats, 0, 4 * sizeof(unsigned long long), st);
    ll_window_kernel<KERN><<<blocks, kWinThreads, 0, st>>>(xs, xy, P, (int)L.pstride, h, m, n, lo, hi, ntiles, nbc,
                                                           ymax, tileS, tileN, counter, stats);
    if (stats) {
        unsigned long long v[4] = {0, 0, 0, 0};
        cudaMemcpyAsync(v, stats, sizeof v, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        cudaFree(stats);
        fprintf(stderr, "ll stats: direct %llu prefix_ok %llu prefix_rejected %llu rejected_window_points %llu\n",
                v[0], v[1], v[2], v[3]);
    }
}

}  // namespace krcv

using namespace krcv;

extern "C" int kr_profile_enable(int on)
{
    g_prof.on = on != 0;
    g_prof.recorded = false;
    return KR_OK;
}

extern "C" int kr_profile_read(float *ms)
{
    if (!ms || !g_prof.recorded) return KR_EARG;
    cudaError_t e = cudaEventSynchronize(g_prof.ev[kProfEvents - 1]);
    if (e != cudaSuccess) { set_cuda_error("cudaEventSynchronize", (int)e); return KR_ECUDA; }
    for (int k = 0; k < kProfEvents - 1; k++) {
        e = cudaEventElapsedTime(&ms[k], g_prof.ev[k], g_prof.ev[k + 1]);
        if (e != cudaSuccess) { set_cuda_error("cudaEventElapsedTime", (int)e); return KR_ECUDA; }
    }
    return KR_OK;
}

extern "C" int64_t kr_launch_count(void) { return g_prof.launches; }

extern "C" int32_t kr_last_algo(void) { return g_prof.algo; }

extern "C" size_t kr_workspace_bytes(int64_t n, int32_t m)
{
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return 0;
    WsLayout L;
    if (!ws_layout(n, m, &L, kWsAll)) return 0;
    return L.total;
}

extern "C" size_t kr_workspace_bytes_algo(int64_t n, int32_t m, int32_t kernel, int32_t algo)
{
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return 0;
    WsLayout L;
    if (!ws_layout(n, m, &L, ws_class_for(algo, kernel, n))) return 0;
    return L.total;
}

extern "C" size_t kr_kde_workspace_bytes(int64_t n, int32_t m)
{
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return 0;
    WsLayout L;
    if (!ws_layout(n, m, &L, kWsKde)) return 0;
    return L.total;
}

// The whole device pipeline of one shard: a1 .. a5, and with fin.cv set the
// fused finalize (single-GPU whole search).
// a1 + a2: validation counters, stable sort of (x, y) by x into the sorted
// AoS array with +-inf sentinels; resets the tile counter.
static int enqueue_sort(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                        const WsLayout &L, char *ws, cudaStream_t st, int64_t *launches_out)
{
    uint64_t *keys_in = reinterpret_cast<uint64_t *>(ws + L.keys_in);
    uint64_t *keys_out = reinterpret_cast<uint64_t *>(ws + L.keys_out);
    uint32_t *vals_in = reinterpret_cast<uint32_t *>(ws + L.vals_in);
    uint32_t *vals_out = reinterpret_cast<uint32_t *>(ws + L.vals_out);
    double2 *xy = reinterpret_cast<double2 *>(ws + L.xy) + kPad;
    int *counter = reinterpret_cast<int *>(ws + L.counter);
    uint32_t *perm = reinterpret_cast<uint32_t *>(ws + L.perm);
    unsigned *status = reinterpret_cast<unsigned *>(ws + L.status);
    const int nn = (int)n;
    int64_t launches = 0;
    cudaError_t e;
    static const int sort_mode = [] {  // KRCV_SORT=cub64 | q32 | rank (A/B runs); KRCV_CUB_SORT=1 = cub64
        const char *e = getenv("KRCV_SORT");
        if (e && strcmp(e, "cub64") == 0) return 1;
        if (e && strcmp(e, "q32") == 0) return 2;
        if (e && strcmp(e, "rank") == 0) return 3;
        return getenv_flag("KRCV_CUB_SORT") ? 1 : 0;
    }();
    const bool use_rank = sort_mode == 3 || (sort_mode == 0 && n <= kRankSortMaxN);
    if (use_rank) {
        // a1 + a2: chunk merge sort, rank by counting across chunk pairs, scatter (krcv_sort.cuh)
        const int cfg = chunk_config(n);
        const int chunk = cfg == 0 ? 1024 : (cfg == 1 ? 2048 : (cfg == 2 ? 4096 : (cfg == 3 ? 512 : 256)));
        const int nchunks = (int)((n + chunk - 1) / chunk);
        uint32_t *khi = reinterpret_cast<uint32_t *>(keys_out);          // keys_out is free on this path
        int *rank = reinterpret_cast<int *>(vals_out);                    // so is vals_out
        switch (cfg) {
        case 0: launch_rank_sort<256, 4>(d_x, d_y, nn, d_h, m, keys_in, khi, vals_in, rank, status, nchunks, st); break;
        case 1: launch_rank_sort<256, 8>(d_x, d_y, nn, d_h, m, keys_in, khi, vals_in, rank, status, nchunks, st); break;
        case 2: launch_rank_sort<512, 8>(d_x, d_y, nn, d_h, m, keys_in, khi, vals_in, rank, status, nchunks, st); break;
        case 3: launch_rank_sort<256, 2>(d_x, d_y, nn, d_h, m, keys_in, khi, vals_in, rank, status, nchunks, st); break;
        default: launch_rank_sort<128, 2>(d_x, d_y, nn, d_h, m, keys_in, khi, vals_in, rank, status, nchunks, st); break;
        }
        const int npad = nchunks * chunk;
        launch_pdl(rank_scatter_kernel, dim3((npad + 255) / 256), dim3(256), 0, st, vals_in, rank, nn, npad, d_x, d_y, xy, perm,
                                                                 counter);
        launches += nchunks > 1 ? 1 : 0;
        launches += 2;
    } else if (sort_mode != 1) {
        // 32-bit quantised keys, 4 radix passes, exact fix-up of equal-key runs (krcv_sort.cuh)
        unsigned long long *kmin_c = reinterpret_cast<unsigned long long *>(ws + L.status + 64);
        unsigned long long *kmax = reinterpret_cast<unsigned long long *>(ws + L.status + 72);
        uint32_t *q_in = reinterpret_cast<uint32_t *>(keys_out);   // free on this path
        uint32_t *q_out = reinterpret_cast<uint32_t *>(keys_in);
        pack_range_kernel<<<grid_for(n, 256), 256, 0, st>>>(d_x, d_y, nn, d_h, m, status, kmin_c, kmax);
        launch_pdl(quant_kernel, dim3(grid_for(n, 256)), dim3(256), 0, st, d_x, nn, (const unsigned long long *)kmin_c,
                   (const unsigned long long *)kmax, q_in, vals_in);
        size_t cub_bytes = L.cub_bytes;
        e = cub::DeviceRadixSort::SortPairs(ws + L.cub, cub_bytes, q_in, q_out, vals_in, vals_out, nn, 0, 32, st);
        if (e != cudaSuccess) { set_cuda_error("cub::DeviceRadixSort::SortPairs", (int)e); return KR_ECUDA; }
        launch_pdl(q32_fixup_kernel, dim3(grid_for(n, 256)), dim3(256), 0, st, d_x, nn, (const uint32_t *)q_out,
                   vals_out);
        launch_pdl(gather_kernel, dim3(grid_for(n, 256)), dim3(256), 0, st, d_x, d_y, vals_out, nn, xy, perm, counter);
        launches += 4 + 2 + 32 / 8;
    } else {
        pack_kernel<<<grid_for(n, 256), 256, 0, st>>>(d_x, d_y, nn, d_h, m, keys_in, vals_in, status);
        size_t cub_bytes = L.cub_bytes;
        e = cub::DeviceRadixSort::SortPairs(ws + L.cub, cub_bytes, keys_in, keys_out, vals_in, vals_out,
                                            nn, 0, 64, st);
        if (e != cudaSuccess) { set_cuda_error("cub::DeviceRadixSort::SortPairs", (int)e); return KR_ECUDA; }
        launch_pdl(gather_kernel, dim3(grid_for(n, 256)), dim3(256), 0, st, d_x, d_y, vals_out, nn, xy, perm, counter);
        launches += 2 + cub_sort_launches(n);
    }
    *launches_out += launches;
    return KR_OK;
}

// reuse_sorted: the workspace already holds this (x, y)'s sorted arrays (and,
// for the window-prefix path, its prefix moments for this kernel) from the
// previous call on it -- only the bandwidth-dependent stages run (the
// coarse-to-fine refinement, kr_cv_refine).
static int enqueue(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                   int32_t algo, int32_t shard, int32_t nshards, double *d_partial, FinOut fin,
                   void *d_workspace, size_t workspace_bytes, void *cuda_stream, bool reuse_sorted = false,
                   bool ll = false, int64_t range_lo = -1, int64_t range_hi = -1)
{
    if (!d_x || !d_y || !d_h || !d_workspace) return KR_EARG;
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (kernel != KR_UNIFORM && kernel != KR_EPANECHNIKOV && kernel != KR_TRIANGULAR && kernel != KR_GAUSSIAN)
        return KR_EKERNEL;
    if (algo != KR_ALGO_AUTO && algo != KR_ALGO_SWEEP && algo != KR_ALGO_PREFIX && algo != KR_ALGO_DENSE &&
        algo != KR_ALGO_HIST)
        return KR_EARG;
    if (ll) {  // local-linear: compact kernels on the window-prefix path only
        if (kernel == KR_GAUSSIAN) return KR_EKERNEL;
        if (algo != KR_ALGO_AUTO && algo != KR_ALGO_PREFIX) return KR_EARG;
        algo = KR_ALGO_PREFIX;
    }
    // the Gaussian has no compact support: only the dense path applies, and
    // the dense path is only for it
    if ((kernel == KR_GAUSSIAN) != (algo == KR_ALGO_DENSE || (algo == KR_ALGO_AUTO && kernel == KR_GAUSSIAN)))
        return KR_EARG;
    const bool ranged = range_lo >= 0;  // explicit rows [range_lo, range_hi) (kr_cv_rows_async)
    if (ranged ? !(range_lo <= range_hi && range_hi <= n) : (nshards < 1 || shard < 0 || shard >= nshards))
        return KR_EARG;
    if ((reinterpret_cast<uintptr_t>(d_workspace) & 255u) != 0) return KR_EARG;
    WsLayout L;
    if (!ws_layout(n, m, &L, ws_class_for(algo, kernel, n))) return KR_ECUDA;
    if (workspace_bytes < L.total) return KR_EARG;

    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    char *ws = static_cast<char *>(d_workspace);
    double2 *xy = reinterpret_cast<double2 *>(ws + L.xy) + kPad;  // first real record
    int *counter = reinterpret_cast<int *>(ws + L.counter);
    double *tileS = reinterpret_cast<double *>(ws + L.tileS);
    uint8_t *tileN = reinterpret_cast<uint8_t *>(ws + L.tileN);
    unsigned *status = reinterpret_cast<unsigned *>(ws + L.status);
    if (!d_partial) d_partial = reinterpret_cast<double *>(ws + L.partial);
    fin.done = status + 2;
    const int nn = (int)n;

    // Rows of this shard in sorted order.
    const int lo = ranged ? (int)range_lo : (int)(((int64_t)shard * n) / nshards);
    const int hi = ranged ? (int)range_hi : (int)(((int64_t)(shard + 1) * n) / nshards);
    if (algo == KR_ALGO_AUTO) algo = kernel == KR_GAUSSIAN ? KR_ALGO_DENSE : auto_algo(n, hi - lo, m, kernel);
    const bool prefix = algo == KR_ALGO_PREFIX;
    const bool dense = algo == KR_ALGO_DENSE;
    const bool hist = algo == KR_ALGO_HIST;
    int hist_warps = 0, hist_mc = m;
    if (hist) {  // shared-memory histogram: warps per CTA that fit 227 KB
        const size_t cap = 227 * 1024;
        for (int w = kHistMaxWarps; w >= 1 && !hist_warps; w--)
            if (hist_smem_bytes(m, w) <= cap) hist_warps = w;
        if (!hist_warps) {  // grid too large for one histogram: slices of the grid, two warps per CTA
            hist_warps = 2;
            hist_mc = (int)(cap / hist_smem_bytes(1, hist_warps));
        }
    }
    const int variant = sweep_variant(hi - lo);
    int G = sweep_G(hi - lo);
    if (variant == 1 && G > 4) G = 4;
    const bool win2 = prefix && !ll && use_win2();  // win_kernel (krcv_window.cuh)
    Win2Shape w2{};
    if (win2) {
        switch (kernel) {
        case KR_UNIFORM: w2 = win2_shape<KR_UNIFORM>(hi - lo, m); break;
        case KR_EPANECHNIKOV: w2 = win2_shape<KR_EPANECHNIKOV>(hi - lo, m); break;
        default: w2 = win2_shape<KR_TRIANGULAR>(hi - lo, m); break;
        }
    }
    const int winK = ll ? 1 : win_rows_per_lane(hi - lo);
    const int rows_per_tile = 32 * win_lane_rows(winK);
    const int ntiles = hist ? (int)((hi - lo + 31) / 32)
                     : win2 ? (w2.ntiles + kWin2Rows - 1) / kWin2Rows  // win_kernel tasks per chunk
                     : prefix ? (int)((hi - lo + rows_per_tile - 1) / rows_per_tile)
                              : dense ? (int)tiles_for(hi - lo, 1)
                                      : (variant == 1 ? (int)tiles_for(hi - lo, 1) : (int)tiles_for(hi - lo, G));

    int64_t launches = 0;
    NvtxScope nv_all("krcv: grid-search shard (a1-a5)");
    prof_mark(0, st);
    // reuse keeps max|y| (words 4-5); the host validated x, y and the grid
    // words 0-7: counters, max|y|, density statistic; bytes 64-79: the key range of the q32 sort
    cudaError_t e = cudaMemsetAsync(status, 0, (reuse_sorted ? 3 : 20) * sizeof(unsigned), st);
    if (e != cudaSuccess) { set_cuda_error("cudaMemsetAsync(status)", (int)e); return KR_ECUDA; }
    if (reuse_sorted) {
        e = cudaMemsetAsync(counter, 0, sizeof(int), st);
        if (e != cudaSuccess) { set_cuda_error("cudaMemsetAsync(counter)", (int)e); return KR_ECUDA; }
    } else {
        if (injected_failure("sort")) return KR_ECUDA;
        NvtxScope nv("krcv: a1+a2 pack, validate, sort");
        const int st2 = enqueue_sort(d_x, d_y, n, d_h, m, L, ws, st, &launches);
        if (st2) return st2;
    }
    prof_mark(1, st);
    if (prefix && !reuse_sorted && injected_failure("prefix")) return KR_ECUDA;
    if (prefix && !reuse_sorted && ll) {
        launch_prefix_build<kLLMoments>(xy, nn, L, ws, st);
        launches += 2;
    } else if (prefix && !reuse_sorted) {
        // win_kernel's bucket table is part of the build (depends on xs only: kept on reuse)
        switch (kernel) {
        case KR_UNIFORM: launches += launch_prefix_build<KR_UNIFORM>(xy, nn, L, ws, st, win2); break;
        case KR_EPANECHNIKOV:
            launches += launch_prefix_build<KR_EPANECHNIKOV>(xy, nn, L, ws, st, win2, lo, hi);
            break;
        default: launches += launch_prefix_build<KR_TRIANGULAR>(xy, nn, L, ws, st, win2); break;
        }
    }
    prof_mark(2, st);
    if (injected_failure("sweep")) return KR_ECUDA;
    if (ntiles > 0) {
        NvtxScope nv("krcv: a3+a4 windows, LOO estimates, squared errors");
        launches += 1;
        if (hist) {
            // Grids larger than one shared-memory histogram run as slices
            // [b0, b0 + mc) of the grid: a neighbour's bucket within a slice is
            // the first of ITS bandwidths whose window holds it (bucket 0 =
            // inside h_b0 already), so each slice's running sums are exactly the
            // full grid's at those bandwidths; the slice writes its rows of the
            // [m][ntiles] partials.  The tile counter is reset between slices.
            const uint32_t *perm = reinterpret_cast<const uint32_t *>(ws + L.perm);
            for (int b0 = 0; b0 < m; b0 += hist_mc) {
                const int mc = m - b0 < hist_mc ? m - b0 : hist_mc;
                if (b0 > 0) {
                    e = cudaMemsetAsync(counter, 0, sizeof(int), st);
                    if (e != cudaSuccess) { set_cuda_error("cudaMemsetAsync(counter)", (int)e); return KR_ECUDA; }
                    launches += 1;
                }
                double *tS = tileS + (size_t)b0 * ntiles;
                uint8_t *tN = tileN + (size_t)b0 * ntiles;
                switch (kernel) {
                case KR_UNIFORM:
                    launch_hist<KR_UNIFORM>(hist_warps, d_x, d_y, perm, xy, d_h + b0, mc, nn, lo, hi, ntiles, tS, tN,
                                            counter, st);
                    break;
                case KR_EPANECHNIKOV:
                    launch_hist<KR_EPANECHNIKOV>(hist_warps, d_x, d_y, perm, xy, d_h + b0, mc, nn, lo, hi, ntiles, tS,
                                                 tN, counter, st);
                    break;
                default:
                    launch_hist<KR_TRIANGULAR>(hist_warps, d_x, d_y, perm, xy, d_h + b0, mc, nn, lo, hi, ntiles, tS,
                                               tN, counter, st);
                    break;
                }
            }
        } else if (dense) {
            const int nrt = (hi - lo + kGThreads - 1) / kGThreads;
            const int nbc = (m + kGB - 1) / kGB;
            gauss_kernel<<<nrt * nbc, kGThreads, 0, st>>>(xy, nn, d_h, m, lo, hi, nbc, ntiles, tileS, tileN);
        } else if (prefix && ll) {
            switch (kernel) {
            case KR_UNIFORM:
                launch_ll_window<KR_UNIFORM>(xy, nn, d_h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st);
                break;
            case KR_EPANECHNIKOV:
                launch_ll_window<KR_EPANECHNIKOV>(xy, nn, d_h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st);
                break;
            default:
                launch_ll_window<KR_TRIANGULAR>(xy, nn, d_h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st);
                break;
            }
        } else if (win2) {
            uint32_t *tileN32 = reinterpret_cast<uint32_t *>(ws + L.tileN);
            switch (kernel) {
            case KR_UNIFORM:
                launch_win2<KR_UNIFORM>(xy, nn, d_h, m, lo, hi, w2, L, ws, tileS, tileN32, st);
                break;
            case KR_EPANECHNIKOV:
                launch_win2<KR_EPANECHNIKOV>(xy, nn, d_h, m, lo, hi, w2, L, ws, tileS, tileN32, st);
                break;
            default:
                launch_win2<KR_TRIANGULAR>(xy, nn, d_h, m, lo, hi, w2, L, ws, tileS, tileN32, st);
                break;
            }
        } else if (prefix) {
            switch (kernel) {
            case KR_UNIFORM:
                launch_window<KR_UNIFORM>(winK, xy, nn, d_h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st);
                break;
            case KR_EPANECHNIKOV:
                launch_window<KR_EPANECHNIKOV>(winK, xy, nn, d_h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st);
                break;
            default:
                launch_window<KR_TRIANGULAR>(winK, xy, nn, d_h, m, lo, hi, ntiles, L, ws, tileS, tileN, counter, st);
                break;
            }
        } else {
            switch (kernel) {
            case KR_UNIFORM:
                launch_sweep<KR_UNIFORM>(G, xy, nn, d_h, m, lo, hi, ntiles, tileS, tileN, counter, st);
                break;
            case KR_EPANECHNIKOV:
                launch_sweep<KR_EPANECHNIKOV>(G, xy, nn, d_h, m, lo, hi, ntiles, tileS, tileN, counter, st);
                break;
            default:
                launch_sweep<KR_TRIANGULAR>(G, xy, nn, d_h, m, lo, hi, ntiles, tileS, tileN, counter, st);
                break;
            }
        }
    }
    prof_mark(3, st);
    if (injected_failure("reduce")) return KR_ECUDA;
    NvtxScope nv_red("krcv: a5 reduction (+ finalize)");
    if (win2)
        launch_pdl(reduce_kernel<uint32_t>, dim3(m < 148 * 8 ? m : 148 * 8), dim3(kReduceThreads), 0, st,
                   (const double *)tileS, (const uint32_t *)(ws + L.tileN), ntiles, m, (const unsigned *)status,
                   d_partial, fin, w2.S, w2.BC);  // tasks per chunk: tile pairs
    else
        launch_pdl(reduce_kernel<uint8_t>, dim3(m < 148 * 8 ? m : 148 * 8), dim3(kReduceThreads), 0, st,
                   (const double *)tileS, (const uint8_t *)tileN, ntiles, m, (const unsigned *)status, d_partial,
                   fin, 0, 0);
    launches += 1;
    prof_mark(4, st);
    g_prof.recorded = g_prof.on;
    g_prof.launches = launches;
    g_prof.algo = algo;
    e = cudaGetLastError();
    if (e != cudaSuccess) { set_cuda_error("kernel launch", (int)e); return KR_ECUDA; }
    return KR_OK;
}

extern "C" int kr_cv_shard_algo_async(const double *d_x, const double *d_y, int64_t n,
                                      const double *d_h, int32_t m, int32_t kernel, int32_t algo,
                                      int32_t shard, int32_t nshards,
                                      double *d_partial, void *d_workspace, size_t workspace_bytes,
                                      void *cuda_stream)
{
    if (!d_partial) return KR_EARG;
    FinOut fin{};
    return enqueue(d_x, d_y, n, d_h, m, kernel, algo, shard, nshards, d_partial, fin, d_workspace,
                   workspace_bytes, cuda_stream);
}

int krcv::enqueue_grid(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                       int32_t kernel, int32_t algo, double *d_cv, int64_t *d_neff, int32_t *d_best_status, void *d_workspace,
                 size_t workspace_bytes, void *cuda_stream, bool reuse_sorted)
{
    if (!d_cv || !d_best_status) return KR_EARG;
    FinOut fin{};
    fin.n = (long long)n;
    fin.cv = d_cv;
    fin.neff = reinterpret_cast<long long *>(d_neff);
    fin.best = d_best_status;
    fin.status = d_best_status + 1;
    return enqueue(d_x, d_y, n, d_h, m, kernel, algo, 0, 1, nullptr, fin, d_workspace, workspace_bytes,
                   cuda_stream, reuse_sorted);
}

extern "C" int kr_cv_grid_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                                int32_t kernel, int32_t algo, double *d_cv, int64_t *d_neff,
                                int32_t *d_best_status, void *d_workspace, size_t workspace_bytes,
                                void *cuda_stream)
{
    return enqueue_grid(d_x, d_y, n, d_h, m, kernel, algo, d_cv, d_neff, d_best_status, d_workspace,
                        workspace_bytes, cuda_stream, false);
}

extern "C" int kr_cv_rows_async(const double *d_x, const double *d_y, int64_t n,
                                const double *d_h, int32_t m, int32_t kernel, int32_t algo,
                                int64_t row_lo, int64_t row_hi,
                                double *d_partial, void *d_workspace, size_t workspace_bytes,
                                void *cuda_stream)
{
    if (!d_partial || row_lo < 0) return KR_EARG;
    FinOut fin{};
    return enqueue(d_x, d_y, n, d_h, m, kernel, algo, 0, 1, d_partial, fin, d_workspace, workspace_bytes,
                   cuda_stream, false, false, row_lo, row_hi);
}

extern "C" int kr_cv_shard_async(const double *d_x, const double *d_y, int64_t n,
                                 const double *d_h, int32_t m, int32_t kernel,
                                 int32_t shard, int32_t nshards,
                                 double *d_partial, void *d_workspace, size_t workspace_bytes,
                                 void *cuda_stream)
{
    return kr_cv_shard_algo_async(d_x, d_y, n, d_h, m, kernel, KR_ALGO_AUTO, shard, nshards, d_partial,
                                  d_workspace, workspace_bytes, cuda_stream);
}

// Local-linear LOO CV (krcv_ll.cuh, reading Q25): same pipeline and
// partial layout as Nadaraya-Watson, other prefix moments and window kernel.
extern "C" int kr_ll_cv_grid_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                                   int32_t kernel, double *d_cv, int64_t *d_neff, int32_t *d_best_status,
                                   void *d_workspace, size_t workspace_bytes, void *cuda_stream)
{
    if (!d_cv || !d_best_status) return KR_EARG;
    FinOut fin{};
    fin.n = (long long)n;
    fin.cv = d_cv;
    fin.neff = reinterpret_cast<long long *>(d_neff);
    fin.best = d_best_status;
    fin.status = d_best_status + 1;
    return enqueue(d_x, d_y, n, d_h, m, kernel, KR_ALGO_PREFIX, 0, 1, nullptr, fin, d_workspace, workspace_bytes,
                   cuda_stream, false, true);
}

extern "C" int kr_ll_shard_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                                 int32_t kernel, int32_t shard, int32_t nshards, double *d_partial,
                                 void *d_workspace, size_t workspace_bytes, void *cuda_stream)
{
    if (!d_partial) return KR_EARG;
    FinOut fin{};
    return enqueue(d_x, d_y, n, d_h, m, kernel, KR_ALGO_PREFIX, shard, nshards, d_partial, fin, d_workspace,
                   workspace_bytes, cuda_stream, false, true);
}

extern "C" int kr_finalize_async(const double *d_partial, int64_t n, int32_t m, double *d_cv,
                                 int64_t *d_neff, int32_t *d_best, int32_t *d_status, void *cuda_stream)
{
    if (!d_partial || !d_cv || !d_best || !d_status || n < 1 || m < 1 || m > KR_MAX_M) return KR_EARG;
    finalize_kernel<<<1, kFinThreads, 0, static_cast<cudaStream_t>(cuda_stream)>>>(
        d_partial, (long long)n, m, d_cv, reinterpret_cast<long long *>(d_neff), d_best, d_status);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { set_cuda_error("finalize_kernel launch", (int)e); return KR_ECUDA; }
    return KR_OK;
}

// ---------------------------------------------------------------------------
// KDE least-squares cross-validation (krcv_kde.cuh; reading Q24)
// ---------------------------------------------------------------------------
static int enqueue_kde(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel, int32_t shard,
                       int32_t nshards, double *d_partial, KdeFin fin, void *d_workspace, size_t workspace_bytes,
                       void *cuda_stream)
{
    if (!d_x || !d_h || !d_workspace) return KR_EARG;
    if (n < 2 || n > 2147483647LL || m < 1 || m > KR_MAX_M) return KR_EARG;
    if (kernel != KR_UNIFORM && kernel != KR_EPANECHNIKOV && kernel != KR_TRIANGULAR) return KR_EKERNEL;
    if (nshards < 1 || shard < 0 || shard >= nshards) return KR_EARG;
    if ((reinterpret_cast<uintptr_t>(d_workspace) & 255u) != 0) return KR_EARG;
    WsLayout L;
    if (!ws_layout(n, m, &L, kWsKde)) return KR_ECUDA;
    if (workspace_bytes < L.total) return KR_EARG;
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    char *ws = static_cast<char *>(d_workspace);
    double2 *xy = reinterpret_cast<double2 *>(ws + L.xy) + kPad;
    int *counter = reinterpret_cast<int *>(ws + L.counter);
    unsigned *status = reinterpret_cast<unsigned *>(ws + L.status);
    double *tileA = reinterpret_cast<double *>(ws + L.tileS);
    double *tileB = reinterpret_cast<double *>(ws + L.tileB);
    if (!d_partial) d_partial = reinterpret_cast<double *>(ws + L.partial);
    fin.done = status + 2;
    const int nn = (int)n;
    const int lo = (int)(((int64_t)shard * n) / nshards);
    const int hi = (int)(((int64_t)(shard + 1) * n) / nshards);
    const int ntiles = (hi - lo + 31) / 32;
    int64_t launches = 0;
    prof_mark(0, st);
    cudaError_t e = cudaMemsetAsync(status, 0, 20 * sizeof(unsigned), st);
    if (e != cudaSuccess) { set_cuda_error("cudaMemsetAsync(status)", (int)e); return KR_ECUDA; }
    // the sort carries (x, y); the density estimate has no y: x rides along
    const int st2 = enqueue_sort(d_x, d_x, n, d_h, m, L, ws, st, &launches);
    if (st2) return st2;
    prof_mark(1, st);
    launch_prefix_build<kKdeMoments>(xy, nn, L, ws, st);
    launches += 2;
    prof_mark(2, st);
    if (ntiles > 0) {
        const int resident = occupancy((const void *)kde_window_kernel<KR_EPANECHNIKOV>, kWinThreads);
        const int sms = dev_info().sms;
        int nbc = (int)(((int64_t)sms * kWinTasksPerSM + ntiles - 1) / ntiles);
        const int max_nbc = (m + kWinMinBper - 1) / kWinMinBper;
        nbc = nbc > max_nbc ? max_nbc : nbc;
        nbc = nbc < 1 ? 1 : nbc;
        int blocks = (int)(((int64_t)ntiles * nbc + kWinWarps - 1) / kWinWarps);
        if (blocks > sms * resident) blocks = sms * resident;
        const double *xs = reinterpret_cast<const double *>(ws + L.xs) + kPad;
        const double *P = reinterpret_cast<const double *>(ws + L.pfx);
        switch (kernel) {
        case KR_UNIFORM:
            kde_window_kernel<KR_UNIFORM><<<blocks, kWinThreads, 0, st>>>(xs, xy, P, (int)L.pstride, d_h, m, nn, lo, hi,
                                                                          ntiles, nbc, tileA, tileB, counter);
            break;
        case KR_EPANECHNIKOV:
            kde_window_kernel<KR_EPANECHNIKOV><<<blocks, kWinThreads, 0, st>>>(xs, xy, P, (int)L.pstride, d_h, m, nn,
                                                                               lo, hi, ntiles, nbc, tileA, tileB,
                                                                               counter);
            break;
        default:
            kde_window_kernel<KR_TRIANGULAR><<<blocks, kWinThreads, 0, st>>>(xs, xy, P, (int)L.pstride, d_h, m, nn, lo,
                                                                             hi, ntiles, nbc, tileA, tileB, counter);
            break;
        }
        launches += 1;
    }
    prof_mark(3, st);
    kde_reduce_kernel<<<m < 148 * 8 ? m : 148 * 8, kKdeRedThreads, 0, st>>>(tileA, tileB, ntiles, m, status,
                                                                             d_partial, fin);
    launches += 1;
    prof_mark(4, st);
    g_prof.recorded = g_prof.on;
    g_prof.launches = launches;
    g_prof.algo = KR_ALGO_PREFIX;
    e = cudaGetLastError();
    if (e != cudaSuccess) { set_cuda_error("kernel launch", (int)e); return KR_ECUDA; }
    return KR_OK;
}

extern "C" int kr_kde_lscv_async(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                                 double *d_lscv, int32_t *d_best_status, void *d_workspace, size_t workspace_bytes,
                                 void *cuda_stream)
{
    if (!d_lscv || !d_best_status) return KR_EARG;
    KdeFin fin{};
    fin.n = (long long)n;
    fin.kernel = kernel;
    fin.h = d_h;
    fin.lscv = d_lscv;
    fin.best = d_best_status;
    fin.status = d_best_status + 1;
    return enqueue_kde(d_x, n, d_h, m, kernel, 0, 1, nullptr, fin, d_workspace, workspace_bytes, cuda_stream);
}

extern "C" int kr_kde_shard_async(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                                  int32_t shard, int32_t nshards, double *d_partial, void *d_workspace,
                                  size_t workspace_bytes, void *cuda_stream)
{
    if (!d_partial) return KR_EARG;
    KdeFin fin{};
    return enqueue_kde(d_x, n, d_h, m, kernel, shard, nshards, d_partial, fin, d_workspace, workspace_bytes,
                       cuda_stream);
}

// ---------------------------------------------------------------------------
// Leave-one-out (jackknife) confidence intervals at the CV-optimal bandwidth
// (krcv_ci.cuh; reading Q26): the grid search, then one launch reading best
// on the device.
// ---------------------------------------------------------------------------
template <bool KDE>
static int enqueue_ci(int64_t n, const double *d_h, int32_t kernel, double *d_est, double *d_se,
                      const int32_t *d_best_status, void *d_workspace, int32_t m, void *cuda_stream)
{
    WsLayout L;  // only the m-independent offsets are read here: any class
    if (!ws_layout(n, m, &L, kWsDefault)) return KR_ECUDA;
    char *ws = static_cast<char *>(d_workspace);
    const double2 *xy = reinterpret_cast<const double2 *>(ws + L.xy) + kPad;
    const uint32_t *perm = reinterpret_cast<const uint32_t *>(ws + L.perm);
    cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
    const dim3 grid((unsigned)((n + kCiThreads - 1) / kCiThreads)), block(kCiThreads);
    const int nn = (int)n;
    switch (kernel) {
    case KR_UNIFORM:
        launch_pdl(ci_kernel<KR_UNIFORM, KDE>, grid, block, 0, st, xy, perm, nn, d_h, d_best_status, d_est, d_se);
        break;
    case KR_EPANECHNIKOV:
        launch_pdl(ci_kernel<KR_EPANECHNIKOV, KDE>, grid, block, 0, st, xy, perm, nn, d_h, d_best_status, d_est,
                   d_se);
        break;
    default:
        launch_pdl(ci_kernel<KR_TRIANGULAR, KDE>, grid, block, 0, st, xy, perm, nn, d_h, d_best_status, d_est, d_se);
        break;
    }
    g_prof.launches += 1;
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) { set_cuda_error("ci_kernel launch", (int)e); return KR_ECUDA; }
    return KR_OK;
}

extern "C" int kr_cv_ci_async(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m,
                              int32_t kernel, double *d_cv, double *d_est, double *d_se, int32_t *d_best_status,
                              void *d_workspace, size_t workspace_bytes, void *cuda_stream)
{
    if (!d_est || !d_se) return KR_EARG;
    if (kernel == KR_GAUSSIAN) return KR_EKERNEL;  // Q26: compact windows
    const int st = enqueue_grid(d_x, d_y, n, d_h, m, kernel, KR_ALGO_AUTO, d_cv, nullptr, d_best_status, d_workspace,
                                workspace_bytes, cuda_stream, false);
    if (st) return st;
    return enqueue_ci<false>(n, d_h, kernel, d_est, d_se, d_best_status, d_workspace, m, cuda_stream);
}

extern "C" int kr_kde_ci_async(const double *d_x, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                               double *d_lscv, double *d_est, double *d_se, int32_t *d_best_status,
                               void *d_workspace, size_t workspace_bytes, void *cuda_stream)
{
    if (!d_est || !d_se) return KR_EARG;
    const int st = kr_kde_lscv_async(d_x, n, d_h, m, kernel, d_lscv, d_best_status, d_workspace, workspace_bytes,
                                     cuda_stream);
    if (st) return st;
    return enqueue_ci<true>(n, d_h, kernel, d_est, d_se, d_best_status, d_workspace, m, cuda_stream);
}
