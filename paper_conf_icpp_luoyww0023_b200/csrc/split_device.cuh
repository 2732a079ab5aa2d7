// split_device.cuh — device helpers shared by the eval and GA translation
// units of the product path (Philox, dexp/Eq. 2, TMA/mbarrier staging, the
// reference cut walk).  Nothing here is shared with oracle/.
#pragma once
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <math_constants.h>
#include <stdint.h>

#include "split_internal.h"

namespace cg = cooperative_groups;

namespace splitga {

constexpr uint32_t NONE = 0xFFFFFFFFu;
#ifdef SPLIT_TRACE_BUILD
constexpr bool kTrace = true;     // phase timestamps (tools: SPLIT_TRACE=<csv>)
#else
constexpr bool kTrace = false;
#endif

// ------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al., SC'11), multipliers/Weyl constants of the
// Random123 reference.  Device-side implementation, independent of oracle/.
// ------------------------------------------------------------------------
__device__ __forceinline__ uint4 philox10(uint4 c, uint32_t k0, uint32_t k1)
{
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
        k0 += 0x9E3779B9u;
        k1 += 0xBB67AE85u;
    }
    return c;
}

__device__ __forceinline__ uint32_t lane_of(const uint4& v, uint32_t l)
{
    return l == 0 ? v.x : (l == 1 ? v.y : (l == 2 ? v.z : v.w));
}

// sequential draws d = 0, 1, ... of one (id, gen, tag) stream
struct Draws {
    uint32_t id, gen, tag, d, k0, k1;
    uint4 blk;
    __device__ __forceinline__ Draws(uint32_t id_, uint32_t gen_, uint32_t tag_, uint32_t k0_, uint32_t k1_)
        : id(id_), gen(gen_), tag(tag_), d(0), k0(k0_), k1(k1_) {}
    __device__ __forceinline__ uint32_t next()
    {
        if ((d & 3u) == 0) blk = philox10(make_uint4(id, gen, tag, d >> 2), k0, k1);
        return lane_of(blk, (d++) & 3u);
    }
};

// uniform integer in [0, m): floor(u * m / 2^32)
__device__ __forceinline__ uint32_t below(uint32_t u, uint32_t m) { return __umulhi(u, m); }

// position of the most significant set bit (one FLO; 0xFFFFFFFF for 0)
__device__ __forceinline__ uint32_t bfind32(uint32_t x)
{
    uint32_t r;
    asm("bfind.u32 %0, %1;" : "=r"(r) : "r"(x));
    return r;
}

// (1 << b) - 1: the bits below position b (one BMSK)
__device__ __forceinline__ uint32_t bmsk32(uint32_t b)
{
    uint32_t r;
    asm("bmsk.clamp.b32 %0, 0, %1;" : "=r"(r) : "r"(b));
    return r;
}

// ------------------------------------------------------------------------
// dexp: exp by the fixed operation sequence of DESIGN.md R5'' (Cody-Waite
// reduction, degree-13 Taylor polynomial in Horner form, RN(1/i!)).
// ------------------------------------------------------------------------
// c_dexp[i] = RN(1/i!) for i = 3..13; [14] = LN2_HI, [15] = LN2_LO
static __constant__ double c_dexp[16] = {
    0.0, 0.0, 0.0,
    0x1.5555555555555p-3,  0x1.5555555555555p-5,  0x1.1111111111111p-7,  0x1.6c16c16c16c17p-10,
    0x1.a01a01a01a01ap-13, 0x1.a01a01a01a01ap-16, 0x1.71de3a556c734p-19, 0x1.27e4fb7789f5cp-22,
    0x1.ae64567f544e4p-26, 0x1.1eed8eff8d898p-29, 0x1.6124613a86d09p-33,
    0x1.62e42fefa39efp-1,  0x1.abc9e3b39803fp-56};
__device__ __forceinline__ double dexp_dev(double z)
{
    if (z > 710.0) return CUDART_INF;
    if (z < -700.0) return 0.0;
    // j = rint(z / ln 2), ties to even: adding 1.5*2^52 rounds to an integer (RN)
    const double t = __dadd_rn(__dmul_rn(z, 0x1.71547652b82fep+0), 0x1.8p52);
    const double j = __dsub_rn(t, 0x1.8p52);
    const int ji = (int)(uint32_t)__double_as_longlong(t);     // low word of t holds j
    // 64-bit constants come from the constant bank (c[3][..] DFMA operands), not
    // from pairs of uniform-register moves
    double r = __fma_rn(-j, c_dexp[14], z);
    r = __fma_rn(-j, c_dexp[15], r);
    double p = c_dexp[13];                      // 1/13!
#pragma unroll
    for (int i = 12; i >= 3; --i) p = __fma_rn(p, r, c_dexp[i]);   // 1/12! .. 1/3!
    p = __fma_rn(p, r, 0.5);
    p = __fma_rn(p, r, 1.0);
    p = __fma_rn(p, r, 1.0);
    // ldexp(p, j) for j in [-2, 1024]: exact scaling by powers of two (p in [0.7, 1.5])
    const int j1 = ji > 1023 ? 1023 : ji;
    const double s1 = __longlong_as_double((long long)(j1 + 1023) << 52);
    const double s2 = __longlong_as_double((long long)(ji - j1 + 1023) << 52);
    return __dmul_rn(__dmul_rn(p, s1), s2);
}

// RN(a/b) for a >= 0, b > 0 (no overflow or underflow) from rb = RN(1/b), in
// five FP64 operations instead of the DDIV sequence.  q0 = RN(a rb) is within
// ~2^-52 relative of a/b; one Newton correction (r = a - b q exactly-enough by
// FMA) brings q within 1/2 ulp + O(2^-104), i.e. faithful; Markstein's theorem
// (rb within 1/2 ulp of 1/b, q faithful => RN(q + (a - b q) rb) = RN(a/b), the
// residual being exact) makes the second correction the correctly rounded
// quotient -- the same value as the oracle's IEEE division (R5').
__device__ __forceinline__ double div_rcp_rn(double a, double b, double rb)
{
    double q = __dmul_rn(a, rb);
    double r = __fma_rn(-b, q, a);
    q = __fma_rn(r, rb, q);
    r = __fma_rn(-b, q, a);
    return __fma_rn(r, rb, q);
}

// Eq. 2 from the exact integer statistics (R5'):
//   x = sigma/T = sqrt(V)/(k T),  y = overhead/m = (OV/T)/k,  f = -(e^(x-1) + e^(y-1))
// rcp: ChainDev::rcp (rcp[0] = RN(1/T), rcp[k] = RN(1/k), rcp[n+1+k] = RN(1/(kT))).
// k T < 2^37 is exact in FP64, so every quotient is the IEEE quotient of the
// same operands the oracle divides.
__device__ __forceinline__ double eq2(uint32_t k, int64_t V, uint64_t OV, uint32_t T, uint32_t n, const double* rcp)
{
    const double rk = __ldg(rcp + k), rkT = __ldg(rcp + n + 1 + k), rT = __ldg(rcp);
    const double Td = __uint2double_rn(T);
    const double kd = __uint2double_rn(k);
    const double x = div_rcp_rn(__dsqrt_rn(__ll2double_rn(V)), __dmul_rn(kd, Td), rkT);
    const double y = div_rcp_rn(div_rcp_rn(__ull2double_rn(OV), Td, rT), kd, rk);
    return -__dadd_rn(dexp_dev(__dsub_rn(x, 1.0)), dexp_dev(__dsub_rn(y, 1.0)));
}
__device__ __forceinline__ double eq2(uint32_t k, int64_t V, uint64_t OV, const ChainDev& ch)
{
    return eq2(k, V, OV, ch.T, ch.n, ch.rcp);
}

__device__ __forceinline__ unsigned long long gtimer()
{
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
// phase timestamps (SPLIT_TRACE): leader CTA 0 slots 0-3, last worker CTA 4-5,
// after the generation barrier 6 (CTA 0) and 7 (last CTA)
__device__ __forceinline__ void trace_mark(const GaArgs& a, uint32_t g, uint32_t slot)
{
    if (!kTrace || !a.trace || threadIdx.x != 0 || blockIdx.x != 0) return;
    const uint32_t gi = g - a.g_begin;
    if (gi < a.trace_gens) a.trace[gi * 16 + slot] = gtimer();
}

// Split grid barrier for the generation loop (all CTAs are co-resident: the
// kernel is a cooperative launch).  arrive: CTA-ordered writes are released at
// gpu scope by one red.release; wait: one thread polls with ld.acquire.
__device__ __forceinline__ void gbar_arrive(unsigned int* ctr)
{
    __syncthreads();
    if (threadIdx.x == 0) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
}
__device__ __forceinline__ void gbar_wait(const unsigned int* ctr, unsigned int target)
{
    if (threadIdx.x == 0) {
        unsigned int v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
        } while ((int)(v - target) < 0);
    }
    __syncthreads();
}

// asynchronous global->shared copies (LDGSTS), no register staging
__device__ __forceinline__ void cp_async8(void* smem_dst, const void* gsrc)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"((uint32_t)__cvta_generic_to_shared(smem_dst)),
                 "l"(gsrc)
                 : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem_dst, const void* gsrc)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"((uint32_t)__cvta_generic_to_shared(smem_dst)),
                 "l"(gsrc)
                 : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// order-preserving u64 key of a fitness (larger f -> larger key)
__device__ __forceinline__ uint64_t fkey(double f)
{
    const uint64_t u = (uint64_t)__double_as_longlong(f);
    return (u >> 63) ? ~u : (u | 0x8000000000000000ull);
}
__device__ __forceinline__ double unkey(uint64_t k)
{
    const uint64_t u = (k >> 63) ? (k & 0x7FFFFFFFFFFFFFFFull) : ~k;
    return __longlong_as_double((long long)u);
}

// ------------------------------------------------------------------------
// Chain staging: one TMA bulk copy of P|ovh into shared memory.
// ------------------------------------------------------------------------
__device__ __forceinline__ void stage_chain(uint32_t* s_chain, const ChainDev& ch, uint64_t* mbar)
{
    const uint32_t bytes = (ch.p_words + ch.o_words) * 4u;   // multiple of 16
    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(mbar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
        const uint32_t dst = (uint32_t)__cvta_generic_to_shared(s_chain);
        const uint32_t chunk = 32768u;
        for (uint32_t off = 0; off < bytes; off += chunk) {
            const uint32_t b = (bytes - off < chunk) ? (bytes - off) : chunk;
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst + off),
                "l"((const char*)ch.words + off), "r"(b), "r"(bar)
                : "memory");
        }
    }
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
            : "=r"(ok)
            : "r"(bar)
            : "memory");
    }
}

// ------------------------------------------------------------------------
// mbarrier + TMA bulk copies (cp.async.bulk) for the leader's loads
// ------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
// shared-memory loads by 32-bit shared address
__device__ __forceinline__ uint32_t lds32(uint32_t a)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
// v = pred ? *a : v, as one predicated load
__device__ __forceinline__ uint32_t lds32_if(bool pred, uint32_t a, uint32_t v)
{
    asm volatile("{ .reg .pred p; setp.ne.u32 p, %2, 0; @p ld.shared.u32 %0, [%1]; }" : "+r"(v) : "r"(a), "r"((uint32_t)pred));
    return v;
}
// a value the compiler must keep in a register (no rematerialisation)
__device__ __forceinline__ uint32_t opaque32(uint32_t x)
{
    asm volatile("mov.u32 %0, %0;" : "+r"(x));
    return x;
}
__device__ __forceinline__ uint2 lds64_if(bool pred, uint32_t a)
{
    uint2 v = make_uint2(0u, 0u);
    asm volatile("{ .reg .pred p; setp.ne.u32 p, %3, 0; @p ld.shared.v2.u32 {%0, %1}, [%2]; }"
                 : "+r"(v.x), "+r"(v.y) : "r"(a), "r"((uint32_t)pred));
    return v;
}
__device__ __forceinline__ uint2 lds64(uint32_t a)
{
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
__device__ __forceinline__ void mbar_init(uint64_t* mbar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(mbar)), "r"(count));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* mbar, uint32_t bytes)
{
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(mbar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* mbar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(mbar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* mbar, uint32_t parity)
{
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
            : "=r"(ok)
            : "r"(smem_u32(mbar)), "r"(parity)
            : "memory");
    }
}
// bytes: multiple of 16; src/dst 16-byte aligned
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* mbar)
{
    const uint32_t d = smem_u32(dst), b = smem_u32(mbar);
    for (uint32_t off = 0; off < bytes; off += 32768u) {
        const uint32_t n = (bytes - off < 32768u) ? (bytes - off) : 32768u;
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d + off),
                     "l"((const char*)src + off), "r"(n), "r"(b)
                     : "memory");
    }
}
// Stage `bytes` (multiple of 16) of global memory into shared memory with TMA
// bulk copies completing on one mbarrier; all threads return after arrival.
__device__ __forceinline__ void stage_bulk(void* s_dst, const void* src, uint32_t bytes, uint64_t* mbar)
{
    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(mbar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
        const uint32_t dst = (uint32_t)__cvta_generic_to_shared(s_dst);
        for (uint32_t off = 0; off < bytes; off += 32768u) {
            const uint32_t b = (bytes - off < 32768u) ? (bytes - off) : 32768u;
            asm volatile(
                "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst + off),
                "l"((const char*)src + off), "r"(b), "r"(bar)
                : "memory");
        }
    }
    uint32_t ok = 0;
    while (!ok) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0, 1, 0, p; }"
            : "=r"(ok)
            : "r"(bar)
            : "memory");
    }
}

// Walk the cuts of one candidate: words come from `get(w)` in ascending order.
// Block j ends at cut c_j; t_j = P[c_j+1] - P[c_{j-1}+1] + ovh[c_{j-1}] (R3).
struct Stats {
    uint32_t k;
    int64_t V;
    uint64_t S1, S2, OV;
};

template <class Get>
__device__ __forceinline__ double eval_walk(const ChainDev& ch, const uint32_t* sP, const uint32_t* sO, Get get,
                                            Stats* st)
{
    uint32_t cuts = 0;
    for (uint32_t w = 0; w < ch.W; ++w) {
        uint64_t v = get(w);
        if (w == ch.W - 1) v &= ch.last_mask;
        cuts += __popcll(v);
    }
    const uint32_t k = cuts + 1;
    if (k < ch.k_min || k > ch.k_max) {
        if (st) st->k = k;
        return -CUDART_INF;
    }
    uint32_t startP = 0, prev_o = 0;
    uint64_t S1 = 0, S2 = 0, OV = 0;
    for (uint32_t w = 0; w < ch.W; ++w) {
        uint64_t v = get(w);
        if (w == ch.W - 1) v &= ch.last_mask;
        while (v) {
            const uint32_t p = w * 64u + (uint32_t)(__ffsll((long long)v) - 1);
            v &= v - 1;
            const uint32_t Pp = sP[p + 1];
            const uint32_t t = Pp - startP + prev_o;
            S1 += t;
            S2 += (uint64_t)t * t;
            prev_o = sO[p];
            OV += prev_o;
            startP = Pp;
        }
    }
    const uint32_t t = ch.T - startP + prev_o;
    S1 += t;
    S2 += (uint64_t)t * t;
    const int64_t V = (int64_t)((uint64_t)k * S2 - S1 * S1);   // exact: V < 2^63 by the a0 guard
    if (st) { st->k = k; st->V = V; st->S1 = S1; st->S2 = S2; st->OV = OV; }
    return eq2(k, V, OV, ch);
}

}  // namespace splitga
