// Microbenchmark: the sync point's small selections (one-warp bitonic of 128 per warp + 16x8
// merge; 512-thread merge sort of <= 512) timed with %globaltimer in each of 148 CTAs.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/microbench_sort tools/microbench_sort.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ bool comp_gt(uint64_t ka, uint32_t ia, uint64_t kb, uint32_t ib)
{
    return ka > kb || (ka == kb && ia < ib);
}
__device__ __forceinline__ unsigned long long gtm() { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ bool gt_nb(uint64_t ka, uint32_t ia, uint64_t kb, uint32_t ib)
{
    return (ka > kb) | ((ka == kb) & (ia < ib));
}

// one warp: bitonic sort of 32*PER entries in registers (entry lane*PER + e) into the
// ranking order of comp_gt; strides below PER inside a lane, the others by shuffles
template <int PER>
__device__ __forceinline__ void warp_bitonic_desc(uint64_t (&k)[PER], uint32_t (&x)[PER], uint32_t lane)
{
    constexpr uint32_t NE = 32u * PER;
#pragma unroll
    for (uint32_t size = 2; size <= NE; size <<= 1) {
#pragma unroll
        for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
            if (stride >= (uint32_t)PER) {                                // across lanes
                const uint32_t pl = stride / PER;
                const bool lower = (lane & pl) == 0u;
                uint64_t ko[PER];
                uint32_t xo[PER];
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    ko[e] = __shfl_xor_sync(0xFFFFFFFFu, k[e], pl);
                    xo[e] = __shfl_xor_sync(0xFFFFFFFFu, x[e], pl);
                }
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    const bool desc = ((lane * PER + e) & size) == 0u;
                    // the lower position of a pair keeps the greater entry when descending (one
                    // compare, flipped by xor: a branch here diverges and serialises the warp; equal
                    // entries are identical sentinels, so swapping them is harmless)
                    const bool take = gt_nb(ko[e], xo[e], k[e], x[e]) != (lower != desc);
                    k[e] = take ? ko[e] : k[e];
                    x[e] = take ? xo[e] : x[e];
                }
            } else {                                                      // inside a lane
#pragma unroll
                for (int e = 0; e < PER; ++e) {
                    if ((e & stride) != 0u) continue;
                    const int f = e | (int)stride;
                    const bool desc = ((lane * PER + e) & size) == 0u;
                    const bool sw = gt_nb(k[f], x[f], k[e], x[e]) == desc;
                    const uint64_t ke = k[e], kf = k[f];
                    const uint32_t xe = x[e], xf = x[f];
                    k[e] = sw ? kf : ke; k[f] = sw ? ke : kf;
                    x[e] = sw ? xf : xe; x[f] = sw ? xe : xf;
                }
            }
        }
    }
}

// one warp: sort entries [0, n) of key/idx (n <= 32*PER); the first m in ranking order to ok/ox
template <int PER>
__device__ __forceinline__ void warp_sort_write(const uint64_t* key, const uint32_t* idx, uint32_t n, uint32_t m,
                                                uint64_t* ok, uint32_t* ox, uint32_t lane)
{
    uint64_t k[PER];
    uint32_t x[PER];
#pragma unroll
    for (int e = 0; e < PER; ++e) {
        const uint32_t j = lane * PER + e;
        k[e] = j < n ? key[j] : 0ull;
        x[e] = j < n ? idx[j] : ~0u;
    }
    warp_bitonic_desc<PER>(k, x, lane);
#pragma unroll
    for (int e = 0; e < PER; ++e) {
        const uint32_t j = lane * PER + e;
        if (j < m) { ok[j] = k[e]; ox[j] = x[e]; }
    }
}

// one warp: the m largest (ranking order) of the union of the lanes' lists -- each lane
// holds PER entries sorted in ranking order -- by m rounds of a butterfly argmax over the
// lanes' heads; the lane whose head won pops it.  The r-th result goes to ok/ox[r].
template <int PER>
__device__ __forceinline__ void warp_topm_lists(uint64_t (&k)[PER], uint32_t (&x)[PER], uint32_t m, uint64_t* ok,
                                                uint32_t* ox, uint32_t lane)
{
    for (uint32_t r = 0; r < m; ++r) {
        uint64_t bk = k[0];
        uint32_t bx = x[0];
#pragma unroll
        for (uint32_t off = 16; off > 0; off >>= 1) {
            const uint64_t ko = __shfl_xor_sync(0xFFFFFFFFu, bk, off);
            const uint32_t xo = __shfl_xor_sync(0xFFFFFFFFu, bx, off);
            const bool take = gt_nb(ko, xo, bk, bx);
            bk = take ? ko : bk;
            bx = take ? xo : bx;
        }
        if (lane == 0) { ok[r] = bk; ox[r] = bx; }
        const bool pop = (k[0] == bk) & (x[0] == bx);    // composites are distinct (sentinels never win)
#pragma unroll
        for (int e = 0; e + 1 < PER; ++e) { k[e] = pop ? k[e + 1] : k[e]; x[e] = pop ? x[e + 1] : x[e]; }
        k[PER - 1] = pop ? 0ull : k[PER - 1];
        x[PER - 1] = pop ? ~0u : x[PER - 1];
    }
}

// All 512 threads: the m largest (m <= 8) of 2048 entries in ranking order: every warp takes the top 8 of its
// 128 (lane-local sort of 4, then warp_topm_lists), one warp the top m of the 16 x 8.
// tk/tx: 128-entry scratch.  The result goes to ok/ox[0..m).
__device__ __forceinline__ void cta_top8_of_2048(const uint64_t* key, const uint32_t* idx, uint32_t m, uint64_t* tk,
                                                 uint32_t* tx, uint64_t* ok, uint32_t* ox)
{
    const uint32_t w = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    {
        uint64_t k[4];
        uint32_t x[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) { k[e] = key[128u * w + 32u * e + lane]; x[e] = idx[128u * w + 32u * e + lane]; }
        // sorting network of 4 inside the lane: (0,1)(2,3)(0,2)(1,3)(1,2)
        auto cx = [&](int a, int b) {
            const bool sw = gt_nb(k[b], x[b], k[a], x[a]);
            const uint64_t ka = k[a], kb = k[b];
            const uint32_t xa = x[a], xb = x[b];
            k[a] = sw ? kb : ka; k[b] = sw ? ka : kb;
            x[a] = sw ? xb : xa; x[b] = sw ? xa : xb;
        };
        cx(0, 1); cx(2, 3); cx(0, 2); cx(1, 3); cx(1, 2);
        warp_topm_lists<4>(k, x, 8u, tk + 8u * w, tx + 8u * w, lane);
    }
    __syncthreads();
    if (w == 0) {
        uint64_t k[8];
        uint32_t x[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            k[e] = lane < 16u ? tk[8u * lane + e] : 0ull;
            x[e] = lane < 16u ? tx[8u * lane + e] : ~0u;
        }
        warp_topm_lists<8>(k, x, m, ok, ox, lane);
    }
    __syncthreads();
}

// All 512 threads: sort n <= 512 entries of key/idx (shared memory) in the ranking order
// and write the first m to ok/ox.  One entry per thread: each warp sorts its 32 by a
// register bitonic network, then four merge levels (runs of 32 -> 512) place every entry
// at its own position plus its rank in the partner run (binary search; the left run wins
// ties, so the sentinels never collide).  bk/bx: 512-entry scratch, distinct from ok/ox
// (key/idx may be one of them).
__device__ void cta_sort512(const uint64_t* key, const uint32_t* idx, uint32_t n, uint32_t m, uint64_t* ok,
                            uint32_t* ox, uint64_t* bk, uint32_t* bx)
{
    const uint32_t lane = threadIdx.x & 31u;
    uint32_t t = threadIdx.x;
    uint64_t k[1];
    uint32_t x[1];
    k[0] = t < n ? key[t] : 0ull;
    x[0] = t < n ? idx[t] : ~0u;
    warp_bitonic_desc<1>(k, x, lane);
    __syncthreads();                             // key/idx may be overwritten below
#pragma unroll
    for (uint32_t L = 32; L < 512; L <<= 1) {
        bk[t] = k[0];
        bx[t] = x[0];
        __syncthreads();
        const uint32_t base = t & ~(2u * L - 1u), pos = t & (L - 1u);
        const bool left = (t & L) == 0u;
        const uint32_t ob = left ? base + L : base;
        // left entries count the partner's strictly greater entries, right entries the
        // greater-or-equal ones (a prefix of the partner run): branch-free binary lifting
        uint32_t lo = 0;
#pragma unroll
        for (uint32_t step = L >> 1; step > 0; step >>= 1) {
            const uint64_t km = bk[ob + lo + step - 1];
            const uint32_t xm = bx[ob + lo + step - 1];
            lo += (gt_nb(km, xm, k[0], x[0]) | (!left & !gt_nb(k[0], x[0], km, xm))) ? step : 0u;
        }
        {
            const uint64_t km = bk[ob + lo];
            const uint32_t xm = bx[ob + lo];
            lo += (gt_nb(km, xm, k[0], x[0]) | (!left & !gt_nb(k[0], x[0], km, xm))) ? 1u : 0u;
        }
        __syncthreads();
        t = base + pos + lo;
    }
    if (t < m) { ok[t] = k[0]; ox[t] = x[0]; }
    __syncthreads();
}


__global__ void __launch_bounds__(512, 1) bench(uint32_t n, int mode, unsigned long long* out, uint32_t* ok)
{
    __shared__ uint64_t k[2048], bk[1024], ok_[1024];
    __shared__ uint32_t ix[2048], bx[1024], ox[1024];
    for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) { k[j] = ((uint64_t)((j + blockIdx.x) * 2654435761u) * 0x9E3779B97F4A7C15ull) >> (j & 7); ix[j] = j; }
    __syncthreads();
    unsigned long long t0 = 0, t1 = 0;
    for (int rep = 0; rep < 2; ++rep) {
        __syncthreads();
        t0 = gtm();
        if (mode == 0) {
            cta_sort512(k, ix, n, n, ok_, ox, bk, bx);
        } else {
            cta_top8_of_2048(k, ix, 8u, bk, bx, ok_, ox);
        }
        t1 = gtm();
    }
    if (threadIdx.x == 0) {
        out[blockIdx.x] = t1 - t0;
        uint32_t good = 1, m = mode == 0 ? n : 8;
        for (uint32_t j = 1; j < m; ++j) good &= !comp_gt(ok_[j], ox[j], ok_[j - 1], ox[j - 1]);
        if (mode == 1) {   // the 8 largest of all 2048
            uint32_t cnt = 0;
            for (uint32_t j = 0; j < n; ++j) cnt += comp_gt(k[j], ix[j], ok_[7], ox[7]) ? 1u : 0u;
            good &= cnt == 7;
        }
        ok[blockIdx.x] = good;
    }
}

int main()
{
    unsigned long long* d; uint32_t* okd;
    cudaMalloc(&d, 8 * 148); cudaMalloc(&okd, 4 * 148);
    struct { uint32_t n; int mode; } cs[] = {{128, 0}, {256, 0}, {448, 0}, {512, 0}, {2048, 1}};
    for (auto c : cs) {
        for (int rep = 0; rep < 5; ++rep) bench<<<148, 512>>>(c.n, c.mode, d, okd);
        unsigned long long h[148]; uint32_t g[148];
        cudaMemcpy(h, d, 8 * 148, cudaMemcpyDeviceToHost); cudaMemcpy(g, okd, 4 * 148, cudaMemcpyDeviceToHost);
        unsigned long long mx = 0, sum = 0; uint32_t allg = 1;
        for (int i = 0; i < 148; ++i) { mx = h[i] > mx ? h[i] : mx; sum += h[i]; allg &= g[i]; }
        printf("%s n=%5u  mean %7.2f us  max %7.2f us  correct=%u\n", c.mode ? "two-level top-8" : "cta_sort512", c.n, sum / 148e3, mx / 1e3, allg);
    }
    return 0;
}
