// Floor of one GA generation on B200: a persistent grid of one 512-thread CTA per
// SM repeating (a) the GA kernel's split grid barrier alone (red.release.gpu arrive,
// ld.acquire.gpu poll, as split_device.cuh gbar_*), and (b) that barrier after two
// dependent L2 round trips per thread (the post-barrier tournament fitness gather,
// then the parent row it selects, from an L2-resident C2-sized population).
// Prints us per iteration.  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/microbench_gridbar tools/microbench_gridbar.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void gbar(unsigned int* ctr, unsigned int target)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
        unsigned int v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
        } while ((int)(v - target) < 0);
    }
    __syncthreads();
}

__global__ void __launch_bounds__(512, 1) k_bar(unsigned int* ctr, const uint64_t* pop, const double* fit,
                                                uint32_t n, int iters, int loads, uint64_t* sink)
{
    unsigned int target = 0;
    uint32_t x = blockIdx.x * 512 + threadIdx.x;
    uint64_t acc = 0;
    for (int it = 0; it < iters; ++it) {
        if (loads) {
            // two dependent L2 round trips: a fitness gather picks the parent row that is loaded next
            x = x * 1664525u + 1013904223u;
            const double f = __ldcg(fit + (x % n));
            const uint32_t parent = (uint32_t)(__double_as_longlong(f) & 0xFFFFFFFu) % n;
            acc += __ldcg(pop + 3ull * parent);
        }
        target += gridDim.x;
        gbar(ctr, target);
    }
    if (acc == 0x123456789ull) sink[0] = acc;
}

int main()
{
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const uint32_t n = 65536;
    unsigned int* ctr; uint64_t* pop; double* fit; uint64_t* sink;
    cudaMalloc(&ctr, 4); cudaMalloc(&pop, 3ull * n * 8); cudaMalloc(&fit, n * 8); cudaMalloc(&sink, 8);
    cudaMemset(pop, 0x5a, 3ull * n * 8); cudaMemset(fit, 0x3f, n * 8);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    for (int loads = 0; loads < 2; ++loads) {
        int iters = 2000;
        void* args[] = {&ctr, &pop, &fit, (void*)&n, &iters, &loads, &sink};
        float best = 1e30f;
        for (int rep = 0; rep < 4; ++rep) {
            cudaMemset(ctr, 0, 4);
            cudaEventRecord(e0);
            cudaLaunchCooperativeKernel((void*)k_bar, dim3(sms), dim3(512), args, 0, 0);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            if (rep > 0 && ms < best) best = ms;
        }
        printf("%s: %.3f us per iteration (%d CTAs x 512 threads)\n",
               loads ? "grid barrier + 2 dependent L2 round trips" : "grid barrier alone", 1000.0f * best / iters, sms);
    }
    return 0;
}
