// Microbenchmark of candidate a2 (ordering step) implementations on B200:
// CUB onesweep radix (u64 key + u32 index), CUB merge sort, single-CTA
// BlockRadixSort.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/sortbench.cu -o /tmp/sortbench
#include <cub/cub.cuh>
#include <cstdio>
#include <vector>
#include <random>
#include <algorithm>

struct KV { unsigned long long k; unsigned v; };
struct LessKV {
    __device__ bool operator()(const unsigned long long &a, const unsigned long long &b) const { return a < b; }
};

template <int THREADS, int ITEMS>
__global__ void __launch_bounds__(THREADS) block_sort(const unsigned long long *kin, const unsigned *vin,
                                                      unsigned long long *kout, unsigned *vout, int n)
{
    using BRS = cub::BlockRadixSort<unsigned long long, THREADS, ITEMS, unsigned, 8>;
    extern __shared__ __align__(16) unsigned char smem[];
    auto &ts = *reinterpret_cast<typename BRS::TempStorage *>(smem);
    unsigned long long k[ITEMS];
    unsigned v[ITEMS];
    for (int i = 0; i < ITEMS; i++) {
        int idx = threadIdx.x * ITEMS + i;
        k[i] = idx < n ? kin[idx] : ~0ull;
        v[i] = idx < n ? vin[idx] : 0u;
    }
    BRS(ts).Sort(k, v);
    for (int i = 0; i < ITEMS; i++) {
        int idx = threadIdx.x * ITEMS + i;
        if (idx < n) { kout[idx] = k[i]; vout[idx] = v[i]; }
    }
}

int main()
{
    for (int n : {20000, 100000, 200000, 1000000}) {
        std::vector<unsigned long long> hk(n);
        std::vector<unsigned> hv(n);
        std::mt19937_64 g(1);
        std::uniform_real_distribution<double> U(0, 1);
        for (int i = 0; i < n; i++) {
            double x = U(g);
            unsigned long long u;
            memcpy(&u, &x, 8);
            hk[i] = u | 0x8000000000000000ull;
            hv[i] = i;
        }
        unsigned long long *dk, *dk2;
        unsigned *dv, *dv2;
        cudaMalloc(&dk, 8 * n); cudaMalloc(&dk2, 8 * n); cudaMalloc(&dv, 4 * n); cudaMalloc(&dv2, 4 * n);
        cudaMemcpy(dk, hk.data(), 8 * n, cudaMemcpyHostToDevice);
        cudaMemcpy(dv, hv.data(), 4 * n, cudaMemcpyHostToDevice);
        size_t tb = 0, tb2 = 0;
        cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dk2, dv, dv2, n);
        cub::DeviceMergeSort::SortPairsCopy(nullptr, tb2, dk, dv, dk2, dv2, n, LessKV());
        void *tmp;
        cudaMalloc(&tmp, std::max(tb, tb2));
        cudaEvent_t a, b;
        cudaEventCreate(&a); cudaEventCreate(&b);
        float ms;
        for (int rep = 0; rep < 3; rep++) cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dk2, dv, dv2, n);
        cudaEventRecord(a);
        for (int rep = 0; rep < 20; rep++) cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dk2, dv, dv2, n);
        cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
        printf("n=%d radix onesweep  %.2f us\n", n, ms * 1000 / 20);
        for (int rep = 0; rep < 3; rep++) cub::DeviceMergeSort::SortPairsCopy(tmp, tb2, dk, dv, dk2, dv2, n, LessKV());
        cudaEventRecord(a);
        for (int rep = 0; rep < 20; rep++) cub::DeviceMergeSort::SortPairsCopy(tmp, tb2, dk, dv, dk2, dv2, n, LessKV());
        cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
        printf("n=%d merge sort      %.2f us\n", n, ms * 1000 / 20);
        for (int bits : {48, 56}) {
            for (int rep = 0; rep < 3; rep++) cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dk2, dv, dv2, n, 64 - bits, 64);
            cudaEventRecord(a);
            for (int rep = 0; rep < 20; rep++) cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dk2, dv, dv2, n, 64 - bits, 64);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            printf("n=%d radix %d bits   %.2f us\n", n, bits, ms * 1000 / 20);
        }
        if (n <= 24576) {
            constexpr int T = 1024, I = 24;
            size_t sm = sizeof(typename cub::BlockRadixSort<unsigned long long, T, I, unsigned, 8>::TempStorage);
            cudaFuncSetAttribute(block_sort<T, I>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            for (int rep = 0; rep < 3; rep++) block_sort<T, I><<<1, T, sm>>>(dk, dv, dk2, dv2, n);
            cudaEventRecord(a);
            for (int rep = 0; rep < 20; rep++) block_sort<T, I><<<1, T, sm>>>(dk, dv, dk2, dv2, n);
            cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b);
            printf("n=%d block radix (1 CTA, smem %zu) %.2f us  err=%s\n", n, sm, ms * 1000 / 20,
                   cudaGetErrorString(cudaGetLastError()));
        }
        cudaFree(dk); cudaFree(dk2); cudaFree(dv); cudaFree(dv2); cudaFree(tmp);
    }
    return 0;
}
