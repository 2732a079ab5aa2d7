// split_exact.cu — SURVEY §8(f) f1: the exact solvers on the GPU.
//
//  * Exhaustive enumeration of all 2^(n-1) splits (n-1 <= kExhMaxPos cut
//    positions).  A cut bitset B is split into its high part Bh (positions
//    >= c) and its low part Bl (positions < c, c = min(6, n-1)).  With
//    H = the lowest cut of Bh (or the chain end) the block times decompose into
//      lower blocks: op 0 .. the cuts of Bl .. cut H   -> a table indexed (H, Bl)
//      upper blocks: cut H .. the cuts of Bh .. end    -> maintained by a Gray walk
//    so each thread walks a range of Gray codes over Bh (one cut toggled per
//    step: O(1) update of the upper-block S2 from the toggled cut's neighbours)
//    and, for every Bh, scans the 2^c table row of its H: k, S1, S2, V and OV
//    of each candidate are a handful of integer adds.  Block times follow R3
//    (the block after cut p pays ovh[p]); V = k S2 - S1^2 exactly (mod 2^64,
//    exact by the create-time guard).
//      MODE_BEST:   the canonical best (f desc, bitset asc) over k in
//                   [k_min, k_max].  Eq. 2 (FP64, R5') is evaluated only for
//                   candidates that pass a necessary condition derived from
//                   the block's best fitness f_b: with y >= 0, f >= f_b needs
//                   e^(x-1) <= -f_b - e^-1, i.e. x, y <= X = 1 + ln(-f_b - e^-1),
//                   i.e. V < (X k T)^2 and OV < X k T (integer thresholds per k,
//                   rounded outwards).  Survivors are compacted per warp and
//                   evaluated 32 at a time.
//      MODE_MINV:   the minimum V per block count k <= k_max.
//      MODE_ARGMIN: the smallest bitset attaining that minimum (canonical).
//  * The O(k n^2) dynamic program for the minimum S2 per block count:
//      D[1][i] = P[i]^2,  D[j][i] = min_{p < i} D[j-1][p] + (P[i] - P[p] + ovh[p-1])^2
//    (block ops p..i-1 starts after the cut at position p-1 and pays its
//    overhead).  With a constant overhead delta, S1 = T + (k-1) delta is fixed
//    and V*_k = k S2*_k - S1^2 is the exact minimum variance of SURVEY §8(c).
#include "split_device.cuh"

namespace splitga {

// one table entry: statistics of the lower blocks of (H, Bl)
struct ExhEntry {
    uint64_t s2;     // sum of the lower blocks' squared times
    uint32_t ov;     // overheads of the cuts of Bl
    uint32_t pc;     // number of cuts in Bl
};

// per-k filter thresholds (MODE_BEST); zero => reject (k out of range)
struct ExhThr {
    uint64_t vmax;
    uint64_t ovmax;
};

struct ExhResult {   // per-CTA result of MODE_BEST
    double f;
    uint64_t bits;
};

__global__ void exh_table_kernel(ExhArgs a)
{
    const uint32_t nb = 1u << a.c, rows = a.m - a.c + 1;
    for (uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x; idx < rows * nb; idx += gridDim.x * blockDim.x) {
        const uint32_t h = a.c + idx / nb, bl = idx % nb;
        uint32_t startB = 0, ov = 0, pc = 0;          // B(-1) = 0: the first block starts at op 0
        uint64_t s2 = 0;
        for (uint32_t p = 0; p < a.c; ++p) {
            if ((bl >> p) & 1u) {
                const uint32_t t = a.A[p] - startB;   // block ..p, after the previous cut
                s2 += (uint64_t)t * t;
                startB = a.B[p];
                ov += a.A[p] - a.B[p];
                ++pc;
            }
        }
        const uint32_t t = a.A[h] - startB;           // last lower block ends at cut H (A[m] = T)
        s2 += (uint64_t)t * t;
        ExhEntry e;
        e.s2 = s2;
        e.ov = ov;
        e.pc = pc;
        ((ExhEntry*)a.tab)[idx] = e;
    }
}

// lowest set bit position of a 64-bit value (x != 0)
__device__ __forceinline__ uint32_t ctz64(uint64_t x) { return (uint32_t)(__ffsll((long long)x) - 1); }
// highest set bit position of a 64-bit value (x != 0)
__device__ __forceinline__ uint32_t msb64(uint64_t x) { return 63u - (uint32_t)__clzll((long long)x); }

// canonical order: (f desc, bits asc)
__device__ __forceinline__ bool exh_better(double fa, uint64_t ba, double fb, uint64_t bb)
{
    return fa > fb || (fa == fb && ba < bb);
}

// Outward-rounded thresholds from a best fitness f_b (MODE_BEST).
__device__ void exh_set_thresholds(const ExhArgs& a, ExhThr* thr, double fb)
{
    // X = 1 + ln(-f_b - e^-1) >= 0; relaxed by a relative and an absolute margin
    const double r = -fb - 0.36787944117144233;
    const double X = (r > 0.0) ? (1.0 + log(r)) * (1.0 + 1e-9) + 1e-12 : 0.0;
    for (uint32_t k = a.k_min; k <= a.k_max; ++k) {
        const double lim = X * (double)k * (double)a.T * (1.0 + 1e-9) + 2.0;   // bound on sqrt(V) and on OV
        const double v2 = lim * lim;
        const uint64_t vmax = (v2 >= 1.8e19) ? ~0ull : (uint64_t)v2 + 1;
        const uint64_t omax = (lim >= 1.8e19) ? ~0ull : (uint64_t)lim + 1;
        if (vmax < thr[k].vmax) atomicMin((unsigned long long*)&thr[k].vmax, (unsigned long long)vmax);
        if (omax < thr[k].ovmax) atomicMin((unsigned long long*)&thr[k].ovmax, (unsigned long long)omax);
    }
}

template <int MODE>
__global__ void __launch_bounds__(kExhThreads) exh_kernel(ExhArgs a)
{
    constexpr uint32_t NW = kExhThreads / 32;
    extern __shared__ __align__(16) uint8_t smem[];
    const uint32_t nb = 1u << a.c, rows = a.m - a.c + 1;
    // [rows][nb + 1]: one pad entry per row shifts each row by 4 banks, so lanes at
    // different lowest high cuts H (different rows, same bl) read different banks
    const uint32_t pitch = nb + 1;
    ExhEntry* s_tab = (ExhEntry*)smem;
    uint32_t* s_A = (uint32_t*)(s_tab + rows * pitch);                    // [m+1]
    uint32_t* s_B = s_A + ((a.m + 1 + 3) & ~3u);                          // [m]
    ExhThr* s_thr = (ExhThr*)(s_B + ((a.m + 3) & ~3u));                   // [65]
    uint64_t* s_kv = (uint64_t*)(s_thr + 65);                             // [65] MINV / ARGMIN
    uint64_t* s_qv = s_kv + 65;                                           // [NW][kExhQ] V
    uint64_t* s_qb = s_qv + NW * kExhQ;                                   // [NW][kExhQ] bits
    uint32_t* s_qo = (uint32_t*)(s_qb + NW * kExhQ);                      // [NW][kExhQ] OV
    uint32_t* s_qk = s_qo + NW * kExhQ;                                   // [NW][kExhQ] k
    ExhResult* s_red = (ExhResult*)(s_qk + NW * kExhQ);                   // [NW]
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;

    for (uint32_t i = tid; i < rows * nb; i += blockDim.x) s_tab[(i / nb) * pitch + i % nb] = ((const ExhEntry*)a.tab)[i];
    for (uint32_t i = tid; i <= a.m; i += blockDim.x) s_A[i] = a.A[i];
    for (uint32_t i = tid; i < a.m; i += blockDim.x) s_B[i] = a.B[i];
    for (uint32_t k = tid; k < 65; k += blockDim.x) {
        const bool in = k >= a.k_min && k <= a.k_max;
        s_thr[k].vmax = in ? ~0ull : 0ull;
        s_thr[k].ovmax = in ? ~0ull : 0ull;
        s_kv[k] = (MODE == MODE_EXH_ARGMIN) ? ~0ull : (MODE == MODE_EXH_MINV ? ~0ull : 0ull);
    }
    __syncthreads();
    if (MODE == MODE_EXH_BEST && tid == 0 && a.seed_f < 0.0) exh_set_thresholds(a, s_thr, a.seed_f);
    if (MODE == MODE_EXH_ARGMIN)    // the minimum V per k of the MINV pass, cached
        for (uint32_t k = tid; k < 65; k += blockDim.x) s_thr[k].vmax = (k <= a.k_max) ? a.kv[k] : ~0ull;
    __syncthreads();

    const uint64_t gt = (uint64_t)blockIdx.x * blockDim.x + tid;
    const uint64_t s0 = gt * a.per_thread;
    uint64_t s1 = s0 + a.per_thread;
    if (s1 > a.outer_total) s1 = a.outer_total;
    const bool active = s0 < s1;

    // state of the high part for Gray index s0
    uint64_t Bh = 0, S2u = 0;
    uint32_t OVu = 0, ku = 0, H = a.m;
    if (active) {
        const uint64_t g0 = s0 ^ (s0 >> 1);
        Bh = g0 << a.c;
        uint64_t rest = Bh;
        if (rest) H = ctz64(rest);
        while (rest) {
            const uint32_t p = ctz64(rest);
            rest &= rest - 1;
            const uint32_t nx = rest ? ctz64(rest) : a.m;
            const uint32_t t = s_A[nx] - s_B[p];
            S2u += (uint64_t)t * t;
            OVu += s_A[p] - s_B[p];
            ++ku;
        }
    }
    double bf = -CUDART_INF;      // this lane's best (MODE_BEST), canonical order
    uint64_t bb = ~0ull;
    uint32_t qn = 0;              // warp queue fill (uniform)
    const uint32_t T = a.T;

    auto flush = [&](uint32_t cnt) {
        __syncwarp();
        if (lane < cnt) {
            const uint32_t e = warp * kExhQ + lane;
            const uint32_t k = s_qk[e];
            const uint64_t V = s_qv[e], bits = s_qb[e];
            const uint32_t OV = s_qo[e];
            const double f = eq2(k, (int64_t)V, OV, T, a.m + 1, a.rcp);
            if (exh_better(f, bits, bf, bb)) {
                bf = f;
                bb = bits;
                // tighten the block's filter (thresholds only decrease: races are harmless)
                exh_set_thresholds(a, s_thr, f);
            }
        }
        __syncwarp();
        // entries beyond 32 move down
        for (uint32_t j = 32 + lane; j < cnt; j += 32) {
            const uint32_t src = warp * kExhQ + j, dst = src - 32;
            s_qk[dst] = s_qk[src];
            s_qv[dst] = s_qv[src];
            s_qb[dst] = s_qb[src];
            s_qo[dst] = s_qo[src];
        }
        __syncwarp();
    };

    const uint32_t c = a.c;
    for (uint64_t s = s0; __any_sync(0xFFFFFFFFu, active && s < s1); ++s) {
        const bool live = active && s < s1;
        const ExhEntry* row = s_tab + (size_t)(H - c) * pitch;
        const uint32_t kb = ku + 1;
        const uint32_t S1b = T + OVu;
        for (uint32_t bl = 0; bl < nb; ++bl) {
            const ExhEntry e = row[bl];
            const uint32_t k = kb + e.pc;
            const uint64_t S2 = S2u + e.s2;
            const uint32_t OV = OVu + e.ov;
            const uint32_t S1 = S1b + e.ov;
            const uint64_t V = (uint64_t)k * S2 - (uint64_t)S1 * S1;
            if (MODE == MODE_EXH_BEST) {
                const ExhThr th = s_thr[k];
                const bool pass = live && V < th.vmax && (uint64_t)OV < th.ovmax;
                const uint32_t bal = __ballot_sync(0xFFFFFFFFu, pass);
                if (bal) {
                    const uint32_t at = qn + __popc(bal & ((1u << lane) - 1u));
                    if (pass) {
                        const uint32_t e2 = warp * kExhQ + at;
                        s_qk[e2] = k;
                        s_qv[e2] = V;
                        s_qb[e2] = Bh | bl;
                        s_qo[e2] = OV;
                    }
                    qn += __popc(bal);
                    if (qn >= 32) {
                        flush(qn);
                        qn -= 32;
                    }
                }
            } else if (MODE == MODE_EXH_MINV) {
                if (live && k <= a.k_max && V < s_kv[k]) atomicMin((unsigned long long*)&s_kv[k], (unsigned long long)V);
            } else {
                if (live && k <= a.k_max && V == s_thr[k].vmax) {
                    const uint64_t bits = Bh | bl;
                    if (bits < s_kv[k]) atomicMin((unsigned long long*)&s_kv[k], (unsigned long long)bits);
                }
            }
        }
        // Gray step s -> s+1: toggle high position c + ctz(s+1)
        if (live && s + 1 < s1) {
            const uint32_t pos = c + ctz64(s + 1);
            const uint64_t bit = 1ull << pos;
            const bool adding = !(Bh & bit);
            const uint64_t below = Bh & (bit - 1);
            const uint64_t above = Bh & ~((bit << 1) - 1);
            const uint32_t hi = above ? ctz64(above) : a.m;
            const uint32_t t2 = s_A[hi] - s_B[pos];              // block (pos, hi]
            const uint64_t q2 = (uint64_t)t2 * t2;
            if (below) {
                const uint32_t lo = msb64(below);
                const uint32_t t0 = s_A[hi] - s_B[lo];           // block (lo, hi] without the cut
                const uint32_t t1 = s_A[pos] - s_B[lo];          // block (lo, pos]
                const uint64_t d = (uint64_t)t1 * t1 + q2 - (uint64_t)t0 * t0;
                S2u = adding ? S2u + d : S2u - d;
            } else {
                // pos is (or was) the lowest high cut H: the upper part gains / loses block (pos, hi]
                S2u = adding ? S2u + q2 : S2u - q2;
                H = adding ? pos : hi;
            }
            const uint32_t o = s_A[pos] - s_B[pos];
            OVu = adding ? OVu + o : OVu - o;
            ku = adding ? ku + 1 : ku - 1;
            Bh ^= bit;
        }
    }
    if (MODE == MODE_EXH_BEST) {
        if (qn) flush(qn);
        // block reduction of the lanes' bests
        for (int off = 16; off > 0; off >>= 1) {
            const double of = __shfl_down_sync(0xFFFFFFFFu, bf, off);
            const uint64_t ob = __shfl_down_sync(0xFFFFFFFFu, bb, off);
            if (exh_better(of, ob, bf, bb)) { bf = of; bb = ob; }
        }
        if (lane == 0) { s_red[warp].f = bf; s_red[warp].bits = bb; }
        __syncthreads();
        if (tid == 0) {
            for (uint32_t w = 1; w < NW; ++w)
                if (exh_better(s_red[w].f, s_red[w].bits, bf, bb)) { bf = s_red[w].f; bb = s_red[w].bits; }
            ExhResult* out = (ExhResult*)a.res;
            out[blockIdx.x].f = bf;
            out[blockIdx.x].bits = bb;
        }
    } else {
        __syncthreads();
        for (uint32_t k = tid; k <= a.k_max && k < 65; k += blockDim.x)
            if (s_kv[k] != ~0ull) atomicMin((unsigned long long*)&a.kv_out[k], (unsigned long long)s_kv[k]);
    }
}

// final reduction of the per-CTA bests (one CTA)
__global__ void exh_reduce_kernel(const ExhResult* res, uint32_t n, ExhResult* out)
{
    double bf = -CUDART_INF;
    uint64_t bb = ~0ull;
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x)
        if (exh_better(res[i].f, res[i].bits, bf, bb)) { bf = res[i].f; bb = res[i].bits; }
    __shared__ ExhResult s[32];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    for (int off = 16; off > 0; off >>= 1) {
        const double of = __shfl_down_sync(0xFFFFFFFFu, bf, off);
        const uint64_t ob = __shfl_down_sync(0xFFFFFFFFu, bb, off);
        if (exh_better(of, ob, bf, bb)) { bf = of; bb = ob; }
    }
    if (lane == 0) { s[warp].f = bf; s[warp].bits = bb; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (uint32_t w = 1; w < (blockDim.x + 31) / 32; ++w)
            if (exh_better(s[w].f, s[w].bits, bf, bb)) { bf = s[w].f; bb = s[w].bits; }
        out->f = bf;
        out->bits = bb;
    }
}

// ------------------------------------------------------------------------
// DP: min S2 per block count, one CTA; D rows in shared memory
// ------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) dp_kernel(const uint32_t* P /*[n+1]*/, const uint32_t* ovh /*[n-1]*/,
                                                 uint32_t n, uint32_t k_max, uint64_t* s2_out /*[k_max+1]*/)
{
    extern __shared__ __align__(16) uint8_t smem[];
    uint64_t* Dp = (uint64_t*)smem;            // [n+1]
    uint64_t* Dc = Dp + (n + 1);               // [n+1]
    uint32_t* sP = (uint32_t*)(Dc + (n + 1));  // [n+1]
    uint32_t* sO = sP + (n + 1);               // [n]: sO[p] = overhead paid by a block starting at op p
    const uint64_t INF = ~0ull;
    for (uint32_t i = threadIdx.x; i <= n; i += blockDim.x) {
        sP[i] = P[i];
        if (i < n) sO[i] = (i == 0) ? 0u : ovh[i - 1];
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i <= n; i += blockDim.x) Dp[i] = (i == 0) ? INF : (uint64_t)sP[i] * sP[i];
    if (threadIdx.x == 0) {
        s2_out[0] = INF;
        if (k_max >= 1) s2_out[1] = (uint64_t)sP[n] * sP[n];
    }
    __syncthreads();
    for (uint32_t j = 2; j <= k_max; ++j) {
        for (uint32_t i = threadIdx.x; i <= n; i += blockDim.x) {
            uint64_t best = INF;
            const uint32_t Pi = sP[i];
            for (uint32_t p = j - 1; p < i; ++p) {
                const uint32_t t = Pi - sP[p] + sO[p];
                const uint64_t v = Dp[p] + (uint64_t)t * t;
                best = (Dp[p] != INF && v < best) ? v : best;
            }
            Dc[i] = best;
        }
        __syncthreads();
        if (threadIdx.x == 0) s2_out[j] = Dc[n];
        uint64_t* tmp = Dp;
        Dp = Dc;
        Dc = tmp;
        __syncthreads();
    }
}

// ------------------------------------------------------------------------
// Two-cut map (f1, the synthetic analog of Fig. 2, P@11560-12128): entry
// [a][b] (a <= b) of the row-major (n-1)^2 outputs is the split with cuts
// {a, b} -- three blocks, or the one-cut split {a} on the diagonal -- with
// its exact V = k S2 - S1^2, OV and Eq. 2 fitness; a > b: V = -1, OV = 0,
// fitness = -inf.  One CTA row per a (blockIdx.y), threads over b: the
// chain pairs {P[b+1], ovh[b]} are read coalesced, the three outputs are
// written coalesced (the kernel is store-bound: 24 B per entry).
// ------------------------------------------------------------------------
__global__ void __launch_bounds__(256) heatmap2_kernel(ChainDev ch, int64_t* __restrict__ var_out,
                                                        uint64_t* __restrict__ ov_out, double* __restrict__ fit_out)
{
    const uint32_t m = ch.n - 1, a = blockIdx.y;
    const uint2 pa = __ldg(ch.po + a);               // {P[a+1], ovh[a]}
    for (uint32_t b = blockIdx.x * blockDim.x + threadIdx.x; b < m; b += gridDim.x * blockDim.x) {
        const size_t e = (size_t)a * m + b;
        int64_t V = -1;
        uint64_t OV = 0;
        double f = -CUDART_INF;
        if (a <= b) {
            const uint2 pb = __ldg(ch.po + b);
            uint32_t k;
            uint64_t S2;
            if (a == b) {                            // one cut: blocks [0, a], [a+1, n-1] (+ ovh[a])
                const uint32_t t1 = pa.x, t2 = ch.T - pa.x + pa.y;
                S2 = (uint64_t)t1 * t1 + (uint64_t)t2 * t2;
                OV = pa.y;
                k = 2;
            } else {                                 // R3: the block after cut p pays ovh[p]
                const uint32_t t1 = pa.x, t2 = pb.x - pa.x + pa.y, t3 = ch.T - pb.x + pb.y;
                S2 = (uint64_t)t1 * t1 + (uint64_t)t2 * t2 + (uint64_t)t3 * t3;
                OV = (uint64_t)pa.y + pb.y;
                k = 3;
            }
            const uint64_t S1 = (uint64_t)ch.T + OV;
            V = (int64_t)((uint64_t)k * S2 - S1 * S1);
            f = eq2(k, V, OV, ch);
        }
        if (var_out) var_out[e] = V;
        if (ov_out) ov_out[e] = OV;
        if (fit_out) fit_out[e] = f;
    }
}

// ------------------------------------------------------------------------
// Launchers
// ------------------------------------------------------------------------
cudaError_t launch_heatmap2(const ChainDev& ch, int64_t* var_out, uint64_t* ov_out, double* fit_out, cudaStream_t st)
{
    const uint32_t m = ch.n - 1;
    const uint32_t gx = (m + 255) / 256;
    heatmap2_kernel<<<dim3(gx, m), 256, 0, st>>>(ch, var_out, ov_out, fit_out);
    return cudaGetLastError();
}

size_t exh_smem_bytes(const ExhArgs& a)
{
    const size_t rows = a.m - a.c + 1, nb = 1u << a.c, NW = kExhThreads / 32;
    return rows * (nb + 1) * sizeof(ExhEntry) + 4 * (((a.m + 1 + 3) & ~3u) + ((a.m + 3) & ~3u)) + 65 * sizeof(ExhThr) +
           65 * 8 + NW * kExhQ * (8 + 8 + 4 + 4) + NW * sizeof(ExhResult);
}

cudaError_t launch_exh_table(const ExhArgs& a, cudaStream_t st)
{
    const uint32_t total = (a.m - a.c + 1) << a.c;
    exh_table_kernel<<<(total + 255) / 256, 256, 0, st>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_exh(const ExhArgs& a, int mode, uint32_t grid, cudaStream_t st)
{
    const size_t sm = exh_smem_bytes(a);
    void* fn = mode == MODE_EXH_BEST ? (void*)exh_kernel<MODE_EXH_BEST>
                                     : (mode == MODE_EXH_MINV ? (void*)exh_kernel<MODE_EXH_MINV> : (void*)exh_kernel<MODE_EXH_ARGMIN>);
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    ExhArgs copy = a;
    void* args[] = {&copy};
    return cudaLaunchKernel(fn, dim3(grid), dim3(kExhThreads), args, sm, st);
}

int exh_blocks_per_sm(const ExhArgs& a)
{
    int per_sm = 0;
    const size_t sm = exh_smem_bytes(a);
    cudaFuncSetAttribute((void*)exh_kernel<MODE_EXH_BEST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (void*)exh_kernel<MODE_EXH_BEST>, kExhThreads, sm);
    return per_sm < 1 ? 1 : per_sm;
}

cudaError_t launch_exh_reduce(const void* res, uint32_t n, void* out, cudaStream_t st)
{
    exh_reduce_kernel<<<1, 1024, 0, st>>>((const ExhResult*)res, n, (ExhResult*)out);
    return cudaGetLastError();
}

cudaError_t launch_dp(const uint32_t* P, const uint32_t* ovh, uint32_t n, uint32_t k_max, uint64_t* s2_out,
                      cudaStream_t st)
{
    const size_t sm = (size_t)(n + 1) * 16 + (size_t)(2 * n + 1) * 4 + 16;
    cudaError_t e = cudaFuncSetAttribute(dp_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    dp_kernel<<<1, 1024, sm, st>>>(P, ovh, n, k_max, s2_out);
    return cudaGetLastError();
}

}  // namespace splitga
