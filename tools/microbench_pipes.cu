// Issue throughput of the instructions on K1's per-cut path (FLO, POPC, BREV,
// IMAD.WIDE, LDS.64, I2F.F64, DFMA) against plain ALU ops, in warp-instructions
// per cycle per SM.  Each thread runs 8 independent chains of (op + IADD); the
// "iadd" row is the same loop with the op replaced by a second ALU op, so the
// difference is the op's own cost.  Tuning aid, not product code.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kChains = 8;

template <int OP>
__global__ void __launch_bounds__(512) k_tp(uint32_t* out, int iters, uint32_t salt)
{
    __shared__ uint2 tab[2048];
    for (int i = threadIdx.x; i < 2048; i += blockDim.x) tab[i] = make_uint2(i * 3u, i * 5u);
    __syncthreads();
    uint32_t a[kChains];
    uint64_t w[kChains];
    double d[kChains];
#pragma unroll
    for (int c = 0; c < kChains; ++c) {
        a[c] = threadIdx.x * 977u + c * 131u + salt;
        w[c] = a[c];
        d[c] = (double)a[c] * 1e-9;
    }
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int c = 0; c < kChains; ++c) {
            uint32_t x = a[c];
            if (OP == 0) { asm volatile("add.u32 %0, %0, %1;" : "+r"(x) : "r"(salt)); }
            if (OP == 1) { uint32_t y; asm volatile("bfind.u32 %0, %1;" : "=r"(y) : "r"(x)); x = y + salt; }
            if (OP == 2) { uint32_t y; asm volatile("popc.b32 %0, %1;" : "=r"(y) : "r"(x)); x = y + salt; }
            if (OP == 3) { uint32_t y; asm volatile("brev.b32 %0, %1;" : "=r"(y) : "r"(x)); x = y + salt; }
            if (OP == 4) { w[c] = (uint64_t)x * x + w[c]; x += salt; }
            if (OP == 5) { const uint2 e = tab[(x + c) & 2047]; x = e.x + e.y + salt; }
            if (OP == 6) { d[c] = __dadd_rn(__uint2double_rn(x), d[c]); x += salt; }
            if (OP == 7) { d[c] = __fma_rn(d[c], 1.0000001, 1e-9); x += salt; }
            if (OP == 8) { uint32_t y; asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(y) : "r"(x), "r"(salt), "r"(i)); x = y + salt; }
            if (OP == 9) { uint32_t y = x * 0x077CB531u; x = (y >> 27) + salt; }
            a[c] = x;
        }
    }
    uint32_t s = 0;
#pragma unroll
    for (int c = 0; c < kChains; ++c) s += a[c] + (uint32_t)w[c] + (uint32_t)(d[c] > 1e300);
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int OP>
float run(uint32_t* out, int blocks, int iters)
{
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    k_tp<OP><<<blocks, 512>>>(out, 16, 1);
    cudaEventRecord(e0);
    k_tp<OP><<<blocks, 512>>>(out, iters, 1);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    return ms;
}

int main()
{
    cudaDeviceProp pr;
    cudaGetDeviceProperties(&pr, 0);
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const int sms = pr.multiProcessorCount, blocks = sms * 4, iters = 4096;
    uint32_t* out;
    cudaMalloc(&out, (size_t)blocks * 512 * 4);
    const char* names[] = {"iadd", "flo(bfind)", "popc", "brev", "imad.wide.u32", "lds.64", "i2f.f64+dadd",
                           "dfma", "lop3", "imul+shr"};
    float ms[10];
    ms[0] = run<0>(out, blocks, iters);
    ms[1] = run<1>(out, blocks, iters);
    ms[2] = run<2>(out, blocks, iters);
    ms[3] = run<3>(out, blocks, iters);
    ms[4] = run<4>(out, blocks, iters);
    ms[5] = run<5>(out, blocks, iters);
    ms[6] = run<6>(out, blocks, iters);
    ms[7] = run<7>(out, blocks, iters);
    ms[8] = run<8>(out, blocks, iters);
    ms[9] = run<9>(out, blocks, iters);
    const double warp_iters = (double)blocks * 16 * iters * kChains;   // per (op + add) pair
    printf("SMs %d  clock %.0f MHz\n", sms, clk_khz / 1e3);
    for (int i = 0; i < 10; ++i) {
        const double cyc = ms[i] * 1e-3 * clk_khz * 1e3;
        printf("%-16s %8.3f ms  %6.3f warp-iter/clk/SM  (%.2f cyc per warp-iter per SMSP)\n", names[i], ms[i],
               warp_iters / cyc / sms, cyc * sms * 4 / warp_iters);
    }
    return 0;
}
