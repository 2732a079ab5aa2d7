// Dependent-chain latencies on the B200 (cycles per op, one warp): DFMA, DDIV,
// DSQRT, FFMA, IMAD.HI (Philox round), LDS, LDG(L2).  Tuning aid, not product code.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_lat(double* dout, uint64_t* tout, const double* gsrc, int iters)
{
    __shared__ uint32_t sbuf[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) sbuf[i] = (i * 7 + 1) & 1023;
    __syncthreads();
    double x = dout[0] + 1.0, y = 1.0000001;
    uint64_t t0, t1;
    // DFMA chain
    t0 = clock64();
    for (int i = 0; i < iters; ++i) x = __fma_rn(x, y, 1e-9);
    t1 = clock64(); tout[0] = (t1 - t0) / iters;
    // DDIV chain
    t0 = clock64();
    for (int i = 0; i < iters; ++i) x = __ddiv_rn(x, 1.0000003);
    t1 = clock64(); tout[1] = (t1 - t0) / iters;
    // DSQRT chain
    t0 = clock64();
    for (int i = 0; i < iters; ++i) x = __dsqrt_rn(x + 2.0);
    t1 = clock64(); tout[2] = (t1 - t0) / iters;
    // FFMA chain
    float fx = (float)x;
    t0 = clock64();
    for (int i = 0; i < iters; ++i) fx = __fmaf_rn(fx, 1.0001f, 1e-6f);
    t1 = clock64(); tout[3] = (t1 - t0) / iters;
    // IMAD.HI + xor (one Philox half-round)
    uint32_t c = (uint32_t)fx;
    t0 = clock64();
    for (int i = 0; i < iters; ++i) c = __umulhi(0xD2511F53u, c) ^ (c * 0xCD9E8D57u) ^ i;
    t1 = clock64(); tout[4] = (t1 - t0) / iters;
    // LDS chain
    uint32_t p = c & 1023;
    t0 = clock64();
    for (int i = 0; i < iters; ++i) p = sbuf[p];
    t1 = clock64(); tout[5] = (t1 - t0) / iters;
    // LDG chain (L2 resident, .cg)
    uint32_t q = p & 255;
    t0 = clock64();
    for (int i = 0; i < iters / 8; ++i) q = (uint32_t)__ldcg(gsrc + q) & 255;
    t1 = clock64(); tout[6] = (t1 - t0) / (iters / 8);
    dout[1] = x + fx + c + p + q;
}

int main()
{
    double* d; uint64_t* t; double* g;
    cudaMalloc(&d, 16); cudaMalloc(&t, 64); cudaMalloc(&g, 256 * 8);
    double h[256];
    for (int i = 0; i < 256; ++i) h[i] = (double)((i * 13 + 5) & 255);
    cudaMemcpy(g, h, sizeof(h), cudaMemcpyHostToDevice);
    cudaMemset(d, 0, 16);
    k_lat<<<1, 32>>>(d, t, g, 4096);
    k_lat<<<1, 32>>>(d, t, g, 4096);
    uint64_t ht[7];
    cudaMemcpy(ht, t, sizeof(ht), cudaMemcpyDeviceToHost);
    const char* names[7] = {"DFMA", "DDIV", "DSQRT", "FFMA", "IMAD.HI^IMAD", "LDS", "LDG.cg(L2)"};
    for (int i = 0; i < 7; ++i) printf("%-14s %llu cycles\n", names[i], (unsigned long long)ht[i]);
    return 0;
}
