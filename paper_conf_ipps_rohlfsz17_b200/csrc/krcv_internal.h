// krcv_internal.h -- declarations shared by the host (krcv_host.cpp) and
// device (krcv_device.cu) halves of libkrcv.so.  Not part of the C-ABI.
#pragma once

#include <cstddef>
#include <cstdint>

namespace krcv {


// Shards with at least this many rows use the gxg sweep variant.
constexpr int64_t kGxgRows = 400000;
int sweep_G(int64_t rows);
int sweep_variant(int64_t rows);
int64_t max_tiles(int64_t n);
// Algorithm for a shard of `rows` rows of an n-point problem when the caller
// asked for KR_ALGO_AUTO.
int auto_algo(int64_t n, int64_t rows, int32_t m, int32_t kernel);

// Byte layout of the device workspace (kr_workspace_bytes / kr_cv_shard_async).
struct WsLayout {
    size_t keys_in, keys_out;   // uint64 [n]  order-preserving keys of x
    size_t vals_in, vals_out;   // uint32 [n]  original indices
    size_t xy;                  // double2 [n + 2 kPad] (x, y) in sorted order, +-inf sentinels
    size_t counter;             // int: sweep tile counter
    size_t perm;                // uint32 [n]  original index of each sorted record (histogram path)
    size_t bt;                  // int32   [Qmax + 1] bucket table of win_kernel (krcv_window.cuh)
    size_t tileS;               // double  [m][ntiles]  per-tile sum of M e^2
    size_t tileN;               // uint8   [m][ntiles]  per-tile sum of M
    size_t tileB;               // double  [m][ceil(n/32)] per-tile KDE sum B (tileS holds A)
    size_t status;              // uint32  [8]  n_bad_grid, n_nonfinite, reduce completion counter, pad,
                                //              u64 bits of max |y| (window-prefix fast-path bound),
                                //              u64 complement bits of the min x-span of kGapSpan+1 records;
                                //              then (byte 32) the BktParams of the call, (bytes 64-79) the
                                //              q32 key range, (bytes 96-223) the anchors' origins o_j
                                //              (anchor_kernel; 256 B region)
    size_t partial;             // double  [2m+2] partial vector of kr_cv_grid_async
    size_t xs;                  // double  [n + 2 kPad] sorted x, +-inf sentinels (prefix path)
    size_t pfx;                 // double [8][2][pstride] dd prefix moments P[k][0..n], hi / lo planes
    size_t ptot;                // double2 [8][nch] prefix tile totals
    size_t pfxa;                // double [5 J pk_slots] anchored hi records of win_kernel, J = anchors_for(n)
                                //        (0 bytes for the sweep / KDE classes, below 50,000 and above kAncMaxN)
    int64_t pstride, nch;
    size_t cub;                 // radix-sort scratch
    size_t cub_bytes;
    size_t total;
    int64_t ntiles_max;
};

// win_kernel's anchors for n points (krcv_window.cuh; 0 = none)
int anchors_for(int64_t n);

// Workspace classes: the partial-sum blocks an algorithm needs (the other
// buffers are common): default = win_kernel slots + one partial per 32-row
// tile (window-prefix, local-linear, dense, histogram, intervals); sweep = +
// the split sweep's 32/G-row tiles; kde = + the KDE sum-B block; all = every
// entry point (kr_workspace_bytes).
enum { kWsDefault = 0, kWsSweep = 1, kWsKde = 2, kWsAll = 3 };
int ws_class_for(int32_t algo, int32_t kernel, int64_t rows);

// Fills `out`; returns false if the CUDA runtime refuses the sort-size query.
bool ws_layout(int64_t n, int32_t m, WsLayout *out, int cls);

// Whole single-GPU search (kr_cv_grid_async) with an optional reuse of the
// sorted arrays / prefix moments already in the workspace (kr_cv_refine).
// Defined outside namespace krcv's anonymous parts, in krcv_device.cu.
int enqueue_grid(const double *d_x, const double *d_y, int64_t n, const double *d_h, int32_t m, int32_t kernel,
                 int32_t algo, double *d_cv, int64_t *d_neff, int32_t *d_best_status, void *d_workspace,
                 size_t workspace_bytes, void *cuda_stream, bool reuse_sorted);

// True while kr_profile_enable(1) is in effect on this thread (the stage
// events must be recorded on a stream, so the host path does not replay a
// captured graph then).
bool prof_enabled();

// Records a CUDA error string for kr_last_cuda_error (thread-local).
void set_cuda_error(const char *what, int code);
void set_error_text(const char *text);

// Fault injection: with KRCV_FAIL_AT=<stage> in the
// environment (stage: sort, prefix, sweep, reduce) the enqueue stops before
// that stage and returns KR_ECUDA, kr_last_cuda_error naming the stage --
// tests/test_gpu_faults.py checks the error unwinding (nothing written, the
// next call clean).  Read per call; unset costs one getenv.
bool injected_failure(const char *stage);

// NVTX range for the host-side enqueue of a stage (nsys / ncu --nvtx);
// header-only NVTX v3, a no-op without an attached tool.
struct NvtxScope {
    explicit NvtxScope(const char *name);
    ~NvtxScope();
    NvtxScope(const NvtxScope &) = delete;
    NvtxScope &operator=(const NvtxScope &) = delete;
};

}  // namespace krcv
