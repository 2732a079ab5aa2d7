// Microbenchmark: in-CTA bitonic sort of n (u64 key, u32 index) pairs in shared memory by 512
// threads -- the GA kernel's leader sort -- timed with %globaltimer inside one CTA.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/microbench_bitonic tools/microbench_bitonic.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ bool comp_gt(uint64_t ka, uint32_t ia, uint64_t kb, uint32_t ib)
{
    return ka > kb || (ka == kb && ia < ib);
}
__device__ __forceinline__ unsigned long long gt() { unsigned long long t; asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t)); return t; }

__device__ void bitonic_desc(uint64_t* k, uint32_t* ix, uint32_t n)
{
    for (uint32_t size = 2; size <= n; size <<= 1) {
        for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
            __syncthreads();
            for (uint32_t t = threadIdx.x; t < n / 2; t += blockDim.x) {
                const uint32_t lo = 2 * t - (t & (stride - 1));
                const uint32_t hi = lo + stride;
                const bool up = (lo & size) == 0;
                const bool g = comp_gt(k[lo], ix[lo], k[hi], ix[hi]);
                if (g != up) {
                    const uint64_t tk = k[lo]; k[lo] = k[hi]; k[hi] = tk;
                    const uint32_t ti = ix[lo]; ix[lo] = ix[hi]; ix[hi] = ti;
                }
            }
        }
    }
    __syncthreads();
}

__global__ void bench(uint32_t n, unsigned long long* out, uint32_t* ok)
{
    __shared__ uint64_t k[4096];
    __shared__ uint32_t ix[4096];
    for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) { k[j] = (uint64_t)(j * 2654435761u) * 0x9E3779B97F4A7C15ull; ix[j] = j; }
    __syncthreads();
    const unsigned long long t0 = gt();
    bitonic_desc(k, ix, n);
    const unsigned long long t1 = gt();
    if (threadIdx.x == 0) {
        out[0] = t1 - t0;
        uint32_t good = 1;
        for (uint32_t j = 1; j < n; ++j) good &= !comp_gt(k[j], ix[j], k[j - 1], ix[j - 1]);
        *ok = good;
    }
}

int main()
{
    unsigned long long* d; uint32_t* ok;
    cudaMalloc(&d, 8); cudaMalloc(&ok, 4);
    for (uint32_t n = 64; n <= 4096; n *= 2) {
        for (int rep = 0; rep < 3; ++rep) bench<<<1, 512>>>(n, d, ok);
        unsigned long long h; uint32_t g;
        cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost); cudaMemcpy(&g, ok, 4, cudaMemcpyDeviceToHost);
        printf("n=%5u  %8.2f us  sorted=%u\n", n, h / 1e3, g);
    }
    return 0;
}
