// fp64_peak.cu -- measured FP64 throughput of this B200 (the roofline
// denominator of the window / sweep / dense kernels; VERDICT r01 "measure
// the FP64 peak on the box").
//
// Every thread runs kChains independent DFMA chains a = fma(a, b, c) for
// `iters` iterations; flops = 2 x chains x iters x threads.  Grid = 148 SMs
// x 8 CTAs x 256 threads (64 warps / SM), enough independent work per
// scheduler to hide the DFMA latency.  A DADD variant (1 flop per
// instruction) gives the add rate.  Built as a shared library
// (libfp64peak.so, exported C entry `fp64_peak_run`) so tools/fp64_peak.py
// can time it with CUDA events under the bench's NVML clock sampler.
#include <cuda_runtime.h>

#include <cstdint>

namespace {
constexpr int kChains = 8;

template <bool FMA>
__global__ void __launch_bounds__(256) fp64_kernel(double *out, int iters, double b, double c)
{
    double a[kChains];
#pragma unroll
    for (int k = 0; k < kChains; k++) a[k] = 1.0 + 1e-3 * (threadIdx.x + k);
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int k = 0; k < kChains; k++) a[k] = FMA ? fma(a[k], b, c) : a[k] + c;
    }
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < kChains; k++) s += a[k];
    if (s == 123.456) out[threadIdx.x] = s;  // never true; keeps the chains live
}
}  // namespace

// Runs `reps` launches of the FMA (fma != 0) or DADD kernel on `stream` and
// returns the best per-launch time in ms through *ms_out, and the flops per
// launch through *flops_out.  0 on success, else the cudaError_t.
extern "C" int fp64_peak_run(int fma, int iters, int reps, void *stream, double *ms_out, double *flops_out)
{
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int blocks = sms * 8, threads = 256;
    double *out = nullptr;
    cudaError_t e = cudaMalloc(&out, sizeof(double) * threads);
    if (e != cudaSuccess) return (int)e;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int r = 0; r < reps + 1; r++) {  // first launch: warm-up
        cudaEventRecord(a, st);
        if (fma)
            fp64_kernel<true><<<blocks, threads, 0, st>>>(out, iters, 0.9999999999, 1e-10);
        else
            fp64_kernel<false><<<blocks, threads, 0, st>>>(out, iters, 0.9999999999, 1e-10);
        cudaEventRecord(b, st);
        cudaEventSynchronize(b);
        float ms = 0.f;
        cudaEventElapsedTime(&ms, a, b);
        if (r > 0 && ms < best) best = ms;
    }
    e = cudaGetLastError();
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    cudaFree(out);
    if (e != cudaSuccess) return (int)e;
    *ms_out = best;
    *flops_out = (double)(fma ? 2 : 1) * kChains * (double)iters * blocks * threads;
    return 0;
}
