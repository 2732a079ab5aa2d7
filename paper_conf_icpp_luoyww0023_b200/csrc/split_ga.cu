// split_ga.cu — the cooperative persistent GA kernel (a1, a3-a9) of SPLIT's
// split search (ICPP'23 §3.3) and its launchers; see DESIGN.md §5.
#include "split_device.cuh"

namespace splitga {

// ------------------------------------------------------------------------
// GA kernel helpers
// ------------------------------------------------------------------------
template <int WT>
struct Row {
    uint64_t w[WT];
};

template <int WT>
__device__ __forceinline__ void row_load(Row<WT>& r, const uint64_t* src, uint32_t W)
{
#pragma unroll
    for (int i = 0; i < WT; ++i) r.w[i] = (i < (int)W) ? src[i] : 0ull;
}
template <int WT>
__device__ __forceinline__ void row_store(const Row<WT>& r, uint64_t* dst, uint32_t W)
{
#pragma unroll
    for (int i = 0; i < WT; ++i)
        if (i < (int)W) dst[i] = r.w[i];
}
// Row words are selected with arithmetic masks, never with a runtime index: an
// indexed access would move the whole row to local memory (ptxas does that to
// if-chains over a runtime word index).
template <int WT>
__device__ __forceinline__ void row_xor_bit(Row<WT>& r, uint32_t p)
{
    const uint32_t wi = p >> 6;
    const uint64_t bit = 1ull << (p & 63);
#pragma unroll
    for (int i = 0; i < WT; ++i) r.w[i] ^= bit & (0ull - (uint64_t)((uint32_t)i == wi));
}
template <int WT>
__device__ __forceinline__ bool row_get_bit(const Row<WT>& r, uint32_t p)
{
    const uint32_t wi = p >> 6;
    uint64_t b = 0;
#pragma unroll
    for (int i = 0; i < WT; ++i) b |= r.w[i] & (0ull - (uint64_t)((uint32_t)i == wi));
    return (b >> (p & 63)) & 1ull;
}
__device__ __forceinline__ uint64_t word_mask(const ChainDev& ch, uint32_t w)
{
    return (w + 1 == ch.W) ? ch.last_mask : ~0ull;
}
// Rows of the GA population never carry padding bits: init, mutation and repair place cuts only
// at positions < n - 1, crossover and migration combine such rows; the register words past W
// are zero (row_load).  So the GA counts and scans rows without masks or W bounds (the padding
// masks stay where external bitsets are read: K1, split_eval.cu).
template <int WT>
__device__ __forceinline__ uint32_t row_popc(const Row<WT>& r, const ChainDev& ch)
{
    uint32_t c = 0;
#pragma unroll
    for (int i = 0; i < WT; ++i)
        c += __popcll(r.w[i]);
    return c;
}

// position of the r-th (0-based) set bit of m (r < popc(m))
__device__ __forceinline__ uint32_t select_bit(uint64_t m, uint32_t r)
{
    uint32_t pos = 0;
    uint32_t c = __popc((uint32_t)m);
    if (r >= c) { r -= c; m >>= 32; pos += 32; }
    uint32_t x = (uint32_t)m;
    c = __popc(x & 0xFFFFu); if (r >= c) { r -= c; x >>= 16; pos += 16; }
    c = __popc(x & 0xFFu);   if (r >= c) { r -= c; x >>= 8;  pos += 8; }
    c = __popc(x & 0xFu);    if (r >= c) { r -= c; x >>= 4;  pos += 4; }
    c = __popc(x & 0x3u);    if (r >= c) { r -= c; x >>= 2;  pos += 2; }
    if (r >= (x & 1u)) pos += 1;
    return pos;
}

// clear (set) the r-th set (unset) valid position, ascending order; unset
// positions below f (front_skip) are not candidates (R22)
template <int WT>
__device__ __forceinline__ void row_toggle_rank(Row<WT>& row, const ChainDev& ch, uint32_t r, bool among_set,
                                                uint32_t f)
{
    // find the word holding the r-th candidate position, then toggle it with a mask
    uint32_t wi = 0xFFFFFFFFu, rr = 0;
    uint64_t mw = 0;
#pragma unroll
    for (int i = 0; i < WT; ++i) {
        if (i < (int)ch.W) {
            const uint32_t lo = 64u * i;
            const uint64_t front = (f <= lo) ? ~0ull : (f >= lo + 64u ? 0ull : ~((1ull << (f - lo)) - 1ull));
            const uint64_t m = (among_set ? row.w[i] : (~row.w[i] & front)) & word_mask(ch, i);
            const uint32_t c = __popcll(m);
            const bool here = (wi == 0xFFFFFFFFu) && r < c;
            wi = here ? (uint32_t)i : wi;
            mw = here ? m : mw;
            rr = here ? r : rr;
            r -= (wi == 0xFFFFFFFFu) ? c : 0u;
        }
    }
    const uint64_t bit = 1ull << select_bit(mw, rr);
#pragma unroll
    for (int i = 0; i < WT; ++i) row.w[i] ^= bit & (0ull - (uint64_t)((uint32_t)i == wi));
}

// Narrow rows (W <= 4): one loop iteration per cut, descending, over the
// row's 32-bit halves held in registers (the next non-empty half is chosen
// from an occupancy mask with a select tree, never with a runtime index), so
// the trip count is the child's cut count rather than a per-word maximum.
// Same integer statistics and Eq. 2 tail as eval_walk (R3, R5').  (The wide form's staged
// {P[p+1], ovh[p]} pairs and the repair's cut count made C2 ~2.5 % slower here: 4.32 vs 4.22 ms
// per 500-generation step; kept for wide rows only.)
template <int WT>
__device__ __forceinline__ double eval_regs_narrow(const ChainDev& ch, const uint32_t* sP, const uint32_t* sO,
                                                   const Row<WT>& r)
{
    constexpr int NH = 2 * WT;
    uint32_t h[NH];
    uint32_t occ = 0, cuts = 0;
#pragma unroll
    for (int i = 0; i < NH; ++i) {
        const uint64_t wv = r.w[i / 2];                 // GA rows: no padding bits (row_popc)
        h[i] = (uint32_t)(wv >> (32 * (i & 1)));
        occ |= (h[i] != 0u ? 1u : 0u) << i;
        cuts += __popc(h[i]);
    }
    const uint32_t k = cuts + 1;
    if (k < ch.k_min || k > ch.k_max) return -CUDART_INF;
    uint32_t endP = ch.T, OV = 0, v = 0, qb = 0;
    uint64_t S2 = 0;
    for (uint32_t j = 0; j < cuts; ++j) {
        if (v == 0u) {
            const uint32_t q = bfind32(occ);
            occ ^= 1u << q;
            // select tree over the halves by the bits of q
            uint32_t t1[NH / 2 > 0 ? NH / 2 : 1];
#pragma unroll
            for (int i = 0; i < NH / 2; ++i) t1[i] = (q & 1u) ? h[2 * i + 1] : h[2 * i];
            if constexpr (NH == 2) v = t1[0];
            else if constexpr (NH == 4) v = (q & 2u) ? t1[1] : t1[0];
            else {
                const uint32_t a0 = (q & 2u) ? t1[1] : t1[0];
                const uint32_t a1 = (q & 2u) ? t1[3] : t1[2];
                v = (q & 4u) ? a1 : a0;
            }
            qb = q << 5;
        }
        const uint32_t bt = bfind32(v);
        v ^= 1u << bt;
        const uint32_t p = qb + bt;
        // the block after cut p runs to the previous (higher) cut and pays ovh[p] (R3)
        const uint32_t Pp = sP[p + 1], op = sO[p];
        const uint32_t t = endP - Pp + op;
        S2 += (uint64_t)t * t;
        OV += op;
        endP = Pp;
    }
    S2 += (uint64_t)endP * endP;                 // first block: ops 0 .. c_1
    const uint64_t S1 = (uint64_t)ch.T + OV;
    const int64_t V = (int64_t)((uint64_t)k * S2 - S1 * S1);
    return eq2(k, V, OV, ch);
}

// Wide rows (4 < W <= 16): the row's 32-bit halves go to this thread's slot of
// shared memory (odd pitch 2W+1: conflict-free), then one loop iteration per
// cut, descending, with a predicated refill from the occupancy mask -- the trip
// count is the child's cut count, not a per-word maximum over the warp's
// lanes.  Same integer statistics and Eq. 2 tail as eval_walk (R3, R5').
template <int WT>
__device__ __forceinline__ double eval_wide(const ChainDev& ch, uint32_t spo_s, const Row<WT>& r, uint32_t* my,
                                            uint32_t cuts)
{
    uint32_t occ = 0;
#pragma unroll
    for (int i = 0; i < WT; ++i) {
        if (i < (int)ch.W) {
            const uint64_t wv = r.w[i];                  // GA rows: no padding bits (row_popc)
            const uint32_t lo = (uint32_t)wv, hi = (uint32_t)(wv >> 32);
            my[2 * i] = lo;
            my[2 * i + 1] = hi;
            occ |= (min(lo, 1u) | (min(hi, 1u) << 1)) << (2 * i);
        }
    }
    const uint32_t k = cuts + 1;
    if (k < ch.k_min || k > ch.k_max) return -CUDART_INF;
    const uint32_t my_s = smem_u32(my);
    uint32_t endP = ch.T, OV = 0, v = 0, tb = spo_s;
    uint64_t S2 = 0;
    for (uint32_t j = 0; j < cuts; ++j) {
        const uint32_t q = bfind32(occ);
        const bool need = (v == 0u);
        occ = need ? (occ & bmsk32(q)) : occ;
        v = lds32_if(need, my_s + 4u * q, v);
        tb = need ? spo_s + (q << 8) : tb;
        const uint32_t bt = bfind32(v);
        v &= bmsk32(bt);
        // the block after cut p runs to the previous (higher) cut and pays ovh[p] (R3)
        const uint2 e = lds64(tb + 8u * bt);
        const uint32_t t = endP - e.x + e.y;
        S2 += (uint64_t)t * t;
        OV += e.y;
        endP = e.x;
    }
    S2 += (uint64_t)endP * endP;                 // first block: ops 0 .. c_1
    const uint64_t S1 = (uint64_t)ch.T + OV;
    const int64_t V = (int64_t)((uint64_t)k * S2 - S1 * S1);
    return eq2(k, V, OV, ch);
}

// spo_s: shared address of the staged {P[p+1], ovh[p]} pairs; cuts_known: the row's
// cut count when the caller has it (else ~0u)
template <int WT>
__device__ __forceinline__ double eval_regs(const ChainDev& ch, const uint32_t* sP, const uint32_t* sO,
                                            const Row<WT>& r, Stats* st, uint32_t* srow = nullptr,
                                            uint32_t spo_s = 0u, uint32_t cuts_known = ~0u)
{
    // (compile-time dispatch: a runtime test here keeps the generic walk below alive in the
    // breeding loop, and its registers cost C2 ~2.4 %: 4.32 vs 4.22 ms per step)
    if constexpr (WT <= 4) {
        if (!st) return eval_regs_narrow<WT>(ch, sP, sO, r);
    } else if constexpr (WT <= 16) {
        if (!st) {
            // wide rows: callers pass srow (this thread's row slot) and spo_s (the staged pairs)
            uint32_t c = cuts_known;
            if (c == ~0u) {
                c = 0;
#pragma unroll
                for (int w = 0; w < WT; ++w)
                    if (w < (int)ch.W) c += __popcll(r.w[w] & word_mask(ch, w));
            }
            return eval_wide<WT>(ch, spo_s, r, srow, c);
        }
    }
    // same arithmetic as eval_walk, with the word loop unrolled over the register row
    uint32_t cuts = 0;
#pragma unroll
    for (int w = 0; w < WT; ++w)
        if (w < (int)ch.W) cuts += __popcll(r.w[w] & word_mask(ch, w));
    const uint32_t k = cuts + 1;
    if (k < ch.k_min || k > ch.k_max) {
        if (st) st->k = k;
        return -CUDART_INF;
    }
    uint32_t startP = 0, prev_o = 0;
    uint64_t S2 = 0, OV = 0;
#pragma unroll
    for (int w = 0; w < WT; ++w) {
        if (w < (int)ch.W) {
            uint64_t v = r.w[w] & word_mask(ch, w);
            while (v) {
                const uint32_t p = 64u * w + (uint32_t)(__ffsll((long long)v) - 1);
                v &= v - 1;
                const uint32_t Pp = sP[p + 1];
                const uint32_t t = Pp - startP + prev_o;
                S2 += (uint64_t)t * t;
                prev_o = sO[p];
                OV += prev_o;
                startP = Pp;
            }
        }
    }
    const uint32_t t = ch.T - startP + prev_o;
    S2 += (uint64_t)t * t;
    const uint64_t S1 = (uint64_t)ch.T + OV;
    const int64_t V = (int64_t)((uint64_t)k * S2 - S1 * S1);
    if (st) { st->k = k; st->V = V; st->S1 = S1; st->S2 = S2; st->OV = OV; }
    return eq2(k, V, OV, ch);
}

// best-record order: (f desc, bitset asc; word W-1 most significant)
__device__ __forceinline__ bool rows_less(const uint64_t* a, const uint64_t* b, uint32_t W)
{
    for (int w = (int)W - 1; w >= 0; --w)
        if (a[w] != b[w]) return a[w] < b[w];
    return false;
}
__device__ __forceinline__ bool better_rec(double fa, uint32_t ia, double fb, uint32_t ib, const uint64_t* base,
                                           uint32_t W)
{
    if (ia == NONE) return false;
    if (ib == NONE) return true;
    if (fa != fb) return fa > fb;
    return rows_less(base + (size_t)ia * W, base + (size_t)ib * W, W);
}

struct BestRef {
    double f;
    uint32_t idx;
};

// block-wide best by (f desc, bits asc) over rows of `base`; all threads call.
__device__ BestRef block_best(BestRef v, const uint64_t* base, uint32_t W, BestRef* scratch)
{
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
#pragma unroll
    for (int off = 16; off; off >>= 1) {
        BestRef o;
        o.f = __shfl_down_sync(0xFFFFFFFFu, v.f, off);
        o.idx = __shfl_down_sync(0xFFFFFFFFu, v.idx, off);
        if (lane + off < 32 && better_rec(o.f, o.idx, v.f, v.idx, base, W)) v = o;
    }
    if (lane == 0) scratch[warp] = v;
    __syncthreads();
    if (warp == 0) {
        v = (lane < nwarps) ? scratch[lane] : BestRef{-CUDART_INF, NONE};
#pragma unroll
        for (int off = 16; off; off >>= 1) {
            BestRef o;
            o.f = __shfl_down_sync(0xFFFFFFFFu, v.f, off);
            o.idx = __shfl_down_sync(0xFFFFFFFFu, v.idx, off);
            if (lane + off < 32 && better_rec(o.f, o.idx, v.f, v.idx, base, W)) v = o;
        }
        if (lane == 0) scratch[32] = v;
    }
    __syncthreads();
    const BestRef r = scratch[32];
    __syncthreads();
    return r;
}

// A candidate best record carried in registers: (f, index, bits).  Ties on f
// are broken on the bits themselves (R10), so no reduction re-reads rows.
template <int WT>
struct BestRow {
    double f;
    uint32_t idx;
    uint32_t pad;
    Row<WT> r;
};

template <int WT>
__device__ __forceinline__ bool better_row(const BestRow<WT>& a, const BestRow<WT>& b, uint32_t W)
{
    if (a.idx == NONE) return false;
    if (b.idx == NONE) return true;
    if (a.f != b.f) return a.f > b.f;
    bool less = false, decided = false;
#pragma unroll
    for (int w = WT - 1; w >= 0; --w)
        if (w < (int)W && !decided && a.r.w[w] != b.r.w[w]) { less = a.r.w[w] < b.r.w[w]; decided = true; }
    return less;
}

template <int WT>
__device__ __forceinline__ BestRow<WT> shfl_down_row(const BestRow<WT>& v, int off, uint32_t W)
{
    BestRow<WT> o;
    o.f = __shfl_down_sync(0xFFFFFFFFu, v.f, off);
    o.idx = __shfl_down_sync(0xFFFFFFFFu, v.idx, off);
    o.pad = 0;
#pragma unroll
    for (int i = 0; i < WT; ++i) o.r.w[i] = (i < (int)W) ? __shfl_down_sync(0xFFFFFFFFu, v.r.w[i], off) : 0ull;
    return o;
}

// block-wide best over BestRow candidates; all threads call; scratch: 33 entries
template <int WT>
__device__ BestRow<WT> block_best_row(BestRow<WT> v, uint32_t W, BestRow<WT>* scratch)
{
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
#pragma unroll
    for (int off = 16; off; off >>= 1) {
        const BestRow<WT> o = shfl_down_row(v, off, W);
        if (lane + off < 32 && better_row(o, v, W)) v = o;
    }
    if (lane == 0) scratch[warp] = v;
    __syncthreads();
    if (warp == 0) {
        if (lane < nwarps) v = scratch[lane];
        else { v.f = -CUDART_INF; v.idx = NONE; }
#pragma unroll
        for (int off = 16; off; off >>= 1) {
            const BestRow<WT> o = shfl_down_row(v, off, W);
            if (lane + off < 32 && better_row(o, v, W)) v = o;
        }
        if (lane == 0) scratch[32] = v;
    }
    __syncthreads();
    const BestRow<WT> r = scratch[32];
    __syncthreads();
    return r;
}

template <int WT>
__device__ __forceinline__ void track_row(BestRow<WT>& b, double f, uint32_t idx, const Row<WT>& r, uint32_t W)
{
    BestRow<WT> c;
    c.f = f;
    c.idx = idx;
    c.pad = 0;
    c.r = r;
    if (better_row(c, b, W)) b = c;
}

template <int WT>
__device__ __forceinline__ void write_partial(const GaArgs& a, size_t slot, const BestRow<WT>& b, uint32_t W)
{
    a.part_f[slot] = b.f;
    a.part_idx[slot] = b.idx;
#pragma unroll
    for (int i = 0; i < WT; ++i)
        if (i < (int)W) a.part_bits[slot * W + i] = b.r.w[i];
}

// composite ranking order (key desc, idx asc)
__device__ __forceinline__ bool comp_gt(uint64_t ka, uint32_t ia, uint64_t kb, uint32_t ib)
{
    return ka > kb || (ka == kb && ia < ib);
}

// bitonic sort of n (power of two) entries in shared memory, descending composite
__device__ void bitonic_desc(uint64_t* k, uint32_t* ix, uint32_t n)
{
    for (uint32_t size = 2; size <= n; size <<= 1) {
        for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
            __syncthreads();
            for (uint32_t t = threadIdx.x; t < n / 2; t += blockDim.x) {
                const uint32_t lo = 2 * t - (t & (stride - 1));
                const uint32_t hi = lo + stride;
                const bool up = (lo & size) == 0;
                const bool gt = comp_gt(k[lo], ix[lo], k[hi], ix[hi]);
                if (gt != up) {
                    const uint64_t tk = k[lo]; k[lo] = k[hi]; k[hi] = tk;
                    const uint32_t ti = ix[lo]; ix[lo] = ix[hi]; ix[hi] = ti;
                }
            }
        }
    }
    __syncthreads();
}

__device__ __forceinline__ uint32_t next_pow2(uint32_t x)
{
    uint32_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

// warp-aggregated append of (key, idx) when pred
__device__ __forceinline__ void append_if(bool pred, uint32_t* cnt, uint64_t* keys, uint32_t* idxs, uint64_t key,
                                          uint32_t idx)
{
    const unsigned act = __activemask();
    const unsigned m = __ballot_sync(act, pred);
    if (!m) return;
    const uint32_t lane = threadIdx.x & 31u;
    const int leader = __ffs(act) - 1;
    uint32_t base = 0;
    if ((int)lane == leader) base = atomicAdd(cnt, (uint32_t)__popc(m));
    base = __shfl_sync(act, base, leader);
    if (pred) {
        const uint32_t r = __popc(m & ((1u << lane) - 1u));
        if (keys) keys[base + r] = key;
        idxs[base + r] = idx;
    }
}

// ------------------------------------------------------------------------
// Shared-memory layout of the GA kernel
// ------------------------------------------------------------------------
struct SelState {
    uint64_t ph;     // resolved prefix of the 96-bit composite (high 64 bits)
    uint32_t pl;     // resolved prefix (low 32 bits)
    uint32_t d;      // resolved digits (0..12)
    uint32_t need;   // elements still to take from the threshold bin
    uint32_t done;
};

struct RecCache {
    double f, f_improve;
    uint32_t valid, gen, last_improve, done;
    uint64_t bits[1];     // W words (allocated to W)
};

struct Smem {
    uint32_t* chain;
    uint64_t* mbar;       // [0]: chain staging, [1]: leader loads (reused every generation), [2]: pair table
    uint2* po;            // staged {P[p+1], ovh[p]} pairs (one LDS.64 per cut in the fused eval)
    uint32_t* hist;       // [I][256]
    SelState* sel;        // [I]
    BestRef* scratch;     // 33 BestRow<WT>
    uint32_t* misc;       // 32 words
    uint32_t* rcw;        // [kRecWin] window of the record-candidate list
    uint64_t* skey;       // [sort_cap]
    uint32_t* sidx;       // [sort_cap]
    uint64_t* ekey;       // [kMaxElite]
    uint64_t* okey;       // [kMaxElite] merged elites (fast path)
    uint32_t* oidx;
    uint32_t* tsel;       // [kMaxElite] in-CTA selection output (sync points)
    RecCache* rec;        // leader: island record + stall state, cached for the whole launch
    double* pf;           // [cpi_pad] staged partial bests (leader)
    uint32_t* pi;
    uint64_t* pb;         // [cpi_pad][W] when a.stage_bits
    uint32_t* rows;       // [kBlock][2W+1] per-thread row halves for the wide-row walk (4 < W <= 16)
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~(size_t)15; }

// register-row width (template WT) used for a row of W words
__host__ __device__ inline uint32_t wt_of(uint32_t W) { return W <= 1 ? 1 : W <= 2 ? 2 : W <= 4 ? 4 : W <= 8 ? 8 : W <= 16 ? 16 : 64; }

__host__ __device__ inline size_t smem_layout(const GaArgs& a, uint8_t* base, Smem* s)
{
    size_t off = 0;
    auto take = [&](size_t bytes) { size_t o = off; off = align16(off + bytes); return base + o; };
    uint8_t* p;
    p = take((size_t)(a.ch.p_words + a.ch.o_words) * 4); if (s) s->chain = (uint32_t*)p;
    p = take(32); if (s) s->mbar = (uint64_t*)p;
    p = take((a.ch.W > 4 && a.ch.W <= 16) ? a.ch.po_bytes : 16); if (s) s->po = (uint2*)p;   // wide rows only
    p = take((size_t)a.I * 256 * 4); if (s) s->hist = (uint32_t*)p;
    p = take((size_t)a.I * sizeof(SelState)); if (s) s->sel = (SelState*)p;
    p = take(33 * (16 + 8 * (size_t)wt_of(a.ch.W))); if (s) s->scratch = (BestRef*)p;
    p = take(128); if (s) s->misc = (uint32_t*)p;
    p = take((size_t)kRecWin * 4); if (s) s->rcw = (uint32_t*)p;
    p = take((size_t)a.sort_cap * 8); if (s) s->skey = (uint64_t*)p;
    p = take((size_t)a.sort_cap * 4); if (s) s->sidx = (uint32_t*)p;
    p = take((size_t)kMaxElite * 8 + 16); if (s) s->ekey = (uint64_t*)p;
    p = take((size_t)kMaxElite * 8); if (s) s->okey = (uint64_t*)p;
    p = take((size_t)kMaxElite * 4); if (s) s->oidx = (uint32_t*)p;
    p = take(sizeof(RecCache) + 8 * (size_t)a.ch.W); if (s) s->rec = (RecCache*)p;
    p = take((size_t)a.cpi_pad * 8); if (s) s->pf = (double*)p;
    p = take(((size_t)a.cpi_pad + 4) * 4); if (s) s->pi = (uint32_t*)p;
    p = take(a.stage_bits ? (size_t)a.cpi_pad * a.ch.W * 8 : 16); if (s) s->pb = (uint64_t*)p;
    p = take((a.ch.W > 4 && a.ch.W <= 16) ? (size_t)kBlock * (2 * a.ch.W + 1) * 4 : 16); if (s) s->rows = (uint32_t*)p;
    p = take((size_t)kMaxElite * 4); if (s) s->tsel = (uint32_t*)p;
    return off;
}

__host__ __device__ inline uint32_t round16(uint32_t bytes) { return (bytes + 15u) & ~15u; }

// composite of element i of an island: desc order (elite/export) -> (key, ~idx);
// worst order (import) -> (~key, idx).  Larger composite = selected first.
__device__ __forceinline__ void composite(double f, uint32_t i, bool worst, uint64_t& hi, uint32_t& lo)
{
    const uint64_t k = fkey(f);
    hi = worst ? ~k : k;
    lo = worst ? i : ~i;
}

__device__ __forceinline__ bool sel_match(uint64_t hi, uint32_t lo, const SelState& s)
{
    if (s.d == 0) return true;
    if (s.d <= 8) return (hi >> (64 - 8 * s.d)) == s.ph;
    if (hi != s.ph) return false;
    const uint32_t dl = s.d - 8;
    return (dl == 4 ? lo : (lo >> (32 - 8 * dl))) == s.pl;
}
__device__ __forceinline__ uint32_t sel_digit(uint64_t hi, uint32_t lo, uint32_t d)
{
    return d < 8 ? (uint32_t)(hi >> (56 - 8 * d)) & 0xFFu : (lo >> (24 - 8 * (d - 8))) & 0xFFu;
}
__device__ __forceinline__ bool sel_selected(uint64_t hi, uint32_t lo, const SelState& s)
{
    if (s.d == 0) return true;
    if (s.d <= 8) return (hi >> (64 - 8 * s.d)) >= s.ph;
    if (hi != s.ph) return hi > s.ph;
    const uint32_t dl = s.d - 8;
    return (dl == 4 ? lo : (lo >> (32 - 8 * dl))) >= s.pl;
}

// General top-Ksel per local island by 96-bit radix select (MSB first, 8-bit
// digits), all CTAs cooperating with grid barriers.  Output (unsorted):
// sel_key/sel_idx[i][0..Ksel) with sel_cnt[i] == Ksel.  fit: [I][Ns].
__device__ void general_select(const GaArgs& a, const double* fit, uint32_t Ksel, bool worst, const Smem& sm,
                               cg::grid_group& grid)
{
    const uint32_t I = a.I, N = a.N;
    for (uint32_t i = threadIdx.x; i < I; i += blockDim.x) {
        SelState s;
        s.ph = 0; s.pl = 0; s.d = 0; s.need = Ksel;
        s.done = (Ksel >= N) || (Ksel == 0);
        sm.sel[i] = s;
    }
    __syncthreads();
    const uint64_t total = (uint64_t)I * N;
    const uint64_t gtid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t gstride = (uint64_t)gridDim.x * blockDim.x;
    uint32_t pass = 0;
    for (;;) {
        bool pending = false;
        for (uint32_t i = 0; i < I; ++i) pending |= !sm.sel[i].done;
        if (!pending) break;
        uint32_t* gh = a.ghist + (size_t)(pass % 3) * I * 256;
        for (uint32_t j = threadIdx.x; j < I * 256; j += blockDim.x) sm.hist[j] = 0;
        __syncthreads();
        for (uint64_t e = gtid; e < total; e += gstride) {
            const uint32_t i = (uint32_t)(e / N), idx = (uint32_t)(e % N);
            const SelState& s = sm.sel[i];
            if (s.done) continue;
            uint64_t hi; uint32_t lo;
            composite(__ldcg(fit + (size_t)i * a.Ns + idx), idx, worst, hi, lo);
            if (sel_match(hi, lo, s)) atomicAdd(&sm.hist[i * 256 + sel_digit(hi, lo, s.d)], 1u);
        }
        __syncthreads();
        for (uint32_t j = threadIdx.x; j < I * 256; j += blockDim.x)
            if (sm.hist[j]) atomicAdd(&gh[j], sm.hist[j]);
        if (blockIdx.x == 0) {
            uint32_t* z = a.ghist + (size_t)((pass + 1) % 3) * I * 256;
            for (uint32_t j = threadIdx.x; j < I * 256; j += blockDim.x) z[j] = 0;
        }
        grid.sync();
        // every CTA derives the same decision from the global histogram
        if (threadIdx.x < 32) {
            for (uint32_t i = 0; i < I; ++i) {
                SelState s = sm.sel[i];
                if (s.done) continue;
                // lane l owns bins 255-8l .. 248-8l (descending)
                const uint32_t lane = threadIdx.x;
                uint32_t c[8], sum = 0;
#pragma unroll
                for (int q = 0; q < 8; ++q) { c[q] = __ldcg(&gh[i * 256 + 255 - 8 * lane - q]); sum += c[q]; }
                // exclusive prefix over lanes (descending bins)
                uint32_t incl = sum;
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, incl, off);
                    if (lane >= (uint32_t)off) incl += o;
                }
                const uint32_t excl = incl - sum;
                const bool mine = excl < s.need && incl >= s.need;
                const unsigned who = __ballot_sync(0xFFFFFFFFu, mine);
                const int src = __ffs(who) - 1;
                uint32_t bin = 0, cnt = 0, before = 0;
                if (mine) {
                    uint32_t acc = excl;
                    for (int q = 0; q < 8; ++q) {
                        if (acc + c[q] >= s.need) { bin = 255 - 8 * lane - q; cnt = c[q]; before = acc; break; }
                        acc += c[q];
                    }
                }
                bin = __shfl_sync(0xFFFFFFFFu, bin, src);
                cnt = __shfl_sync(0xFFFFFFFFu, cnt, src);
                before = __shfl_sync(0xFFFFFFFFu, before, src);
                if (lane == 0) {
                    s.need -= before;
                    if (s.d < 8) s.ph = (s.ph << 8) | bin;
                    else s.pl = (s.pl << 8) | bin;
                    s.d += 1;
                    if (cnt == s.need || s.d == 12) s.done = 1;
                    sm.sel[i] = s;
                }
                __syncwarp();
            }
        }
        __syncthreads();
        ++pass;
    }
    // compaction: exactly Ksel per island satisfy sel_selected
    for (uint64_t e = gtid; e < total; e += gstride) {
        const uint32_t i = (uint32_t)(e / N), idx = (uint32_t)(e % N);
        const SelState s = sm.sel[i];
        const double f = __ldcg(fit + (size_t)i * a.Ns + idx);
        uint64_t hi; uint32_t lo;
        composite(f, idx, worst, hi, lo);
        const bool take = (Ksel > 0) && sel_selected(hi, lo, s);
        if (take) {
            const uint32_t slot = atomicAdd(&a.sel_cnt[i], 1u);
            a.sel_key[(size_t)i * kMaxElite + slot] = fkey(f);
            a.sel_idx[(size_t)i * kMaxElite + slot] = idx;
        }
    }
    grid.sync();
    if (blockIdx.x == 0) {
        for (uint32_t j = threadIdx.x; j < 3 * I * 256; j += blockDim.x) a.ghist[j] = 0;
    }
}

// ------------------------------------------------------------------------
// In-CTA selection (one leader CTA, all its threads): the k largest of n
// (key, idx) entries in shared memory under the ranking order of comp_gt
// (key desc, idx asc), by an MSB radix select over the 96-bit composite
// (key, ~idx) -- a few passes of a 256-bin shared histogram, starting below
// the key bytes every entry shares; no sort of the n entries (an in-CTA
// bitonic sort of 2048 entries costs ~29 us on B200,
// tools/microbench_bitonic.cu; a one-warp select was slower still: its
// histogram atomics serialise) -- then the k selected are ordered by rank
// counting into ok/ox[0..k).  hist: 256 words, st: one SelState, counter:
// one word, tk/tx: >= k scratch; all in shared memory; k <= 1024.
// ------------------------------------------------------------------------
__device__ void cta_select_sorted(const uint64_t* key, const uint32_t* idx, uint32_t n, uint32_t k, uint32_t* hist,
                                  SelState* st, uint32_t* counter, uint64_t* tk, uint32_t* tx, uint64_t* ok,
                                  uint32_t* ox)
{
    // leading bytes of the key that every entry shares need no pass: the select starts below them
    if (threadIdx.x == 0) { hist[0] = 0; hist[1] = 0; *counter = 0; }
    __syncthreads();
    const uint64_t k0 = n ? key[0] : 0ull;
    uint64_t diff = 0;
    for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) diff |= key[j] ^ k0;
#pragma unroll
    for (int off = 16; off; off >>= 1) diff |= __shfl_xor_sync(0xFFFFFFFFu, diff, off);
    if ((threadIdx.x & 31u) == 0 && diff) {
        atomicOr(hist, (uint32_t)(diff >> 32));
        atomicOr(hist + 1, (uint32_t)diff);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const uint64_t dall = ((uint64_t)hist[0] << 32) | hist[1];
        const uint32_t d0 = dall ? (uint32_t)__clzll((long long)dall) / 8u : 8u;   // 0..8 common bytes
        st->ph = d0 == 0 ? 0ull : (d0 >= 8 ? k0 : (k0 >> (64 - 8 * d0)));
        st->pl = 0;
        st->d = d0;
        st->need = k;
        st->done = (k >= n) || (k == 0);
    }
    __syncthreads();
    while (!st->done) {
        for (uint32_t j = threadIdx.x; j < 256; j += blockDim.x) hist[j] = 0;
        __syncthreads();
        const SelState s = *st;
        for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) {
            const uint64_t hi = key[j];
            const uint32_t lo = ~idx[j];
            if (sel_match(hi, lo, s)) atomicAdd(&hist[sel_digit(hi, lo, s.d)], 1u);
        }
        __syncthreads();
        if (threadIdx.x < 32) {
            const uint32_t lane = threadIdx.x;
            uint32_t c[8], sum = 0;
#pragma unroll
            for (int q = 0; q < 8; ++q) { c[q] = hist[255 - 8 * lane - q]; sum += c[q]; }
            uint32_t incl = sum;
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, incl, off);
                if (lane >= (uint32_t)off) incl += o;
            }
            const uint32_t excl = incl - sum;
            const bool mine = excl < s.need && incl >= s.need;
            const int src = __ffs(__ballot_sync(0xFFFFFFFFu, mine)) - 1;
            uint32_t bin = 0, cnt = 0, before = 0;
            if (mine) {
                uint32_t acc = excl;
                for (int q = 0; q < 8; ++q) {
                    if (acc + c[q] >= s.need) { bin = 255 - 8 * lane - q; cnt = c[q]; before = acc; break; }
                    acc += c[q];
                }
            }
            bin = __shfl_sync(0xFFFFFFFFu, bin, src);
            cnt = __shfl_sync(0xFFFFFFFFu, cnt, src);
            before = __shfl_sync(0xFFFFFFFFu, before, src);
            if (lane == 0) {
                SelState t = s;
                t.need -= before;
                if (t.d < 8) t.ph = (t.ph << 8) | bin;
                else t.pl = (t.pl << 8) | bin;
                t.d += 1;
                if (cnt == t.need || t.d == 12) t.done = 1;
                *st = t;
            }
        }
        __syncthreads();
    }
    // the selected entries (exactly min(k, n)) to tk/tx, then ordered by rank counting
    const SelState s = *st;
    const bool all = k >= n;
    for (uint32_t j = threadIdx.x; j < n; j += blockDim.x) {
        if (all || sel_selected(key[j], ~idx[j], s)) {
            const uint32_t p = atomicAdd(counter, 1u);
            if (p < k) { tk[p] = key[j]; tx[p] = idx[j]; }
        }
    }
    __syncthreads();
    const uint32_t m = min(*counter, k);
    for (uint32_t j = threadIdx.x; j < m; j += blockDim.x) {
        const uint64_t kj = tk[j];
        const uint32_t xj = tx[j];
        uint32_t r = 0;
        for (uint32_t q = 0; q < m; ++q) r += comp_gt(tk[q], tx[q], kj, xj) ? 1u : 0u;
        ok[r] = kj;
        ox[r] = xj;
    }
    __syncthreads();
}

// ------------------------------------------------------------------------
// Small selections (sync points): sorts instead of the radix select, which
// pays ~1.2 us per 8-bit digit and needs up to 12 digits when the keys of a
// converged island tie.  Branch-free compares (the branchy form serialises on
// every shuffle).  Sentinel entries (key 0, idx ~0) sort last: no fitness key
// is 0.
// ------------------------------------------------------------------------
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

// All threads (>= 512; 16 warps work): the m largest (m <= 8) of 2048 entries in ranking order: every warp takes the top 8 of its
// 128 (lane-local sort of 4, then warp_topm_lists), one warp the top m of the 16 x 8.
// tk/tx: 128-entry scratch.  The result goes to ok/ox[0..m).
__device__ __forceinline__ void cta_top8_of_2048(const uint64_t* key, const uint32_t* idx, uint32_t m, uint64_t* tk,
                                                 uint32_t* tx, uint64_t* ok, uint32_t* ox)
{
    const uint32_t w = threadIdx.x >> 5, lane = threadIdx.x & 31u;
    if (w < 16u) {
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

// All threads (>= 512; the first 512 work): sort n <= 512 entries of key/idx (shared memory) in the ranking order
// and write the first m to ok/ox.  One entry per thread: each warp sorts its 32 by a
// register bitonic network, then four merge levels (runs of 32 -> 512) place every entry
// at its own position plus its rank in the partner run (binary search; the left run wins
// ties, so the sentinels never collide).  bk/bx: 512-entry scratch, distinct from ok/ox
// (key/idx may be one of them).
__device__ void cta_sort512(const uint64_t* key, const uint32_t* idx, uint32_t n, uint32_t m, uint64_t* ok,
                            uint32_t* ox, uint64_t* bk, uint32_t* bx)
{
    const uint32_t lane = threadIdx.x & 31u;
    const bool act = threadIdx.x < 512u;        // whole warps: the shuffles below stay warp-uniform
    uint32_t t = threadIdx.x;
    uint64_t k[1];
    uint32_t x[1];
    k[0] = t < n ? key[t] : 0ull;
    x[0] = t < n ? idx[t] : ~0u;
    warp_bitonic_desc<1>(k, x, lane);
    __syncthreads();                             // key/idx may be overwritten below
#pragma unroll
    for (uint32_t L = 32; L < 512; L <<= 1) {
        if (act) {
            bk[t] = k[0];
            bx[t] = x[0];
        }
        __syncthreads();
        const uint32_t base = t & ~(2u * L - 1u), pos = t & (L - 1u);
        const bool left = (t & L) == 0u;
        const uint32_t ob = left ? base + L : base;
        // left entries count the partner's strictly greater entries, right entries the
        // greater-or-equal ones (a prefix of the partner run): branch-free binary lifting
        uint32_t lo = 0;
        if (act) {
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
        }
        __syncthreads();
        t = base + pos + lo;
    }
    if (act && t < m) { ok[t] = k[0]; ox[t] = x[0]; }
    __syncthreads();
}

// The k largest of n entries in ranking order to ok/ox[0..min(k, n)) -- the same result
// as cta_select_sorted (composites are distinct): the merge sort above when n <= 512 and
// the CTA has 512 threads, the radix select otherwise.  All threads of the CTA call it;
// the inputs must be visible (a __syncthreads after they were written).  sm.okey/oidx
// serve as scratch, as they do for the radix select.
__device__ __forceinline__ void select_sorted(const uint64_t* key, const uint32_t* idx, uint32_t n, uint32_t k,
                                           const Smem& sm, uint64_t* ok, uint32_t* ox)
{
    if (n > 512u || blockDim.x < 512u) {
        cta_select_sorted(key, idx, n, k, sm.hist, sm.sel, sm.misc + 4, sm.okey, sm.oidx, ok, ox);
        return;
    }
    cta_sort512(key, idx, n, min(k, n), ok, ox, sm.okey, sm.oidx);
}

// Leader CTA: sort the general-select output of island i in smem (ranking
// order, or worst order) and leave it in sm.skey/sm.sidx[0..Ksel).
__device__ void leader_sort_selected(const GaArgs& a, uint32_t i, uint32_t Ksel, bool worst, const Smem& sm)
{
    const uint32_t P2 = next_pow2(Ksel < 2 ? 2 : Ksel);
    for (uint32_t j = threadIdx.x; j < P2; j += blockDim.x) {
        if (j < Ksel) {
            const uint64_t k = a.sel_key[(size_t)i * kMaxElite + j];
            const uint32_t x = a.sel_idx[(size_t)i * kMaxElite + j];
            sm.skey[j] = worst ? ~k : k;
            sm.sidx[j] = worst ? ~x : x;
        } else {
            sm.skey[j] = 0;
            sm.sidx[j] = NONE;
        }
    }
    bitonic_desc(sm.skey, sm.sidx, P2);
    if (worst)
        for (uint32_t j = threadIdx.x; j < Ksel; j += blockDim.x) { sm.skey[j] = ~sm.skey[j]; sm.sidx[j] = ~sm.sidx[j]; }
    __syncthreads();
    if (threadIdx.x == 0) a.sel_cnt[i] = 0;
}


// Leader CTA: load island i's record and stall state into shared memory once
// per launch; every update writes through to global memory for the host.
__device__ void rec_load(const GaArgs& a, uint32_t i, const Smem& sm)
{
    if (threadIdx.x == 0) {
        RecCache* r = sm.rec;
        r->valid = __ldcg(a.rec_valid + i);
        r->f = __ldcg(a.rec_f + i);
        r->gen = __ldcg(a.rec_gen + i);
        for (uint32_t w = 0; w < a.ch.W; ++w) r->bits[w] = __ldcg(a.rec_bits + (size_t)i * a.ch.W + w);
        r->f_improve = __ldcg(&a.ctl->f_improve);
        r->last_improve = __ldcg(&a.ctl->last_improve);
        r->done = 0;
    }
    __syncthreads();
}

// thread-level best over this thread's share of the per-CTA partials, from global
template <int WT>
__device__ __forceinline__ BestRow<WT> load_partials(const GaArgs& a, uint32_t i, uint32_t parity)
{
    const uint32_t W = a.ch.W;
    BestRow<WT> v;
    v.f = -CUDART_INF;
    v.idx = NONE;
    const size_t base = ((size_t)parity * a.I + i) * a.cpi_pad;
    for (uint32_t j = threadIdx.x; j < a.cpi; j += blockDim.x) {
        BestRow<WT> o;
        o.f = __ldcg(a.part_f + base + j);
        o.idx = __ldcg(a.part_idx + base + j);
#pragma unroll
        for (int w = 0; w < WT; ++w) o.r.w[w] = (w < (int)W) ? __ldcg(a.part_bits + (base + j) * W + w) : 0ull;
        if (better_row(o, v, W)) v = o;
    }
    return v;
}

// Record update of island i with the best candidate of generation g (block-
// reduced when `reduce`), the single-island stall rule (R11), and the snapshot
// of the record that breed(g+1) filters against.
template <int WT>
__device__ void record_apply(const GaArgs& a, uint32_t i, uint32_t g, BestRow<WT> v, bool reduce, const Smem& sm)
{
    const uint32_t W = a.ch.W;
    if (reduce) v = block_best_row(v, W, (BestRow<WT>*)sm.scratch);
    if (threadIdx.x == 0) {
        RecCache* rc = sm.rec;
        bool upd = false;
        if (reduce && v.idx != NONE) {
            if (!rc->valid) upd = true;
            else if (v.f != rc->f) upd = v.f > rc->f;
            else {
                BestRow<WT> rec;
                rec.f = v.f;
                rec.idx = 0;
#pragma unroll
                for (int w = 0; w < WT; ++w) rec.r.w[w] = (w < (int)W) ? rc->bits[w] : 0ull;
                upd = better_row(v, rec, W);
            }
        }
        if (upd) {
            rc->f = v.f;
            rc->gen = g;
            rc->valid = 1;
            a.rec_f[i] = v.f;
            a.rec_gen[i] = g;
            a.rec_valid[i] = 1;
#pragma unroll
            for (int w = 0; w < WT; ++w)
                if (w < (int)W) { rc->bits[w] = v.r.w[w]; a.rec_bits[(size_t)i * W + w] = v.r.w[w]; }
        }
        // snapshot of generation g's record for breed(g+1) (parity g&1)
        const uint32_t sp = (g & 1u) * a.I + i;
        a.snap_f[sp] = rc->valid ? rc->f : -CUDART_INF;
        for (uint32_t w = 0; w < W; ++w) a.snap_bits[(size_t)sp * W + w] = rc->valid ? rc->bits[w] : ~0ull;
        if (a.stall_in_kernel && i == 0) {
            if (g == 0) {
                rc->f_improve = rc->f;
                rc->last_improve = 0;
            } else {
                if (rc->f > rc->f_improve) { rc->f_improve = rc->f; rc->last_improve = g; }
                if (a.stall > 0 && g - rc->last_improve >= a.stall) { rc->done = 1; a.ctl->done = 1; }
            }
            a.ctl->f_improve = rc->f_improve;
            a.ctl->last_improve = rc->last_improve;
        }
    }
    __syncthreads();
}

// INIT: record of generation 0 from the per-CTA partial bests; both snapshots
template <int WT>
__device__ void leader_record(const GaArgs& a, uint32_t i, uint32_t g, uint32_t parity, const Smem& sm)
{
    record_apply<WT>(a, i, g, load_partials<WT>(a, i, parity), true, sm);
    if (threadIdx.x == 0) {
        const uint32_t sp = (1u - (g & 1u)) * a.I + i;
        a.snap_f[sp] = a.snap_f[(g & 1u) * a.I + i];
        for (uint32_t w = 0; w < a.ch.W; ++w)
            a.snap_bits[(size_t)sp * a.ch.W + w] = a.snap_bits[((size_t)(g & 1u) * a.I + i) * a.ch.W + w];
    }
}

// Record of generation g from the record-candidate list (children that beat a
// snapshot of an earlier record, list g%3).  R entries, the first kRecWin of
// them staged in sm.rcw; rows and fitness are read from generation g.
template <int WT>
__device__ __forceinline__ BestRow<WT> rec_list_best(const GaArgs& a, uint32_t i, uint32_t g, uint32_t R, bool staged,
                                                     const Smem& sm)
{
    const uint32_t W = a.ch.W, L = g % 3u, cur = g & 1u;
    const uint64_t* popc = a.pop[cur] + (size_t)i * a.N * W;
    const double* fitc = a.fit[cur] + (size_t)i * a.Ns;
    const uint32_t* lst = a.rc_idx[L] + (size_t)i * a.Ns;
    BestRow<WT> v;
    v.f = -CUDART_INF;
    v.idx = NONE;
    for (uint32_t r = threadIdx.x; r < R; r += blockDim.x) {
        const uint32_t slot = (staged && r < kRecWin) ? sm.rcw[r] : __ldcg(lst + r);
        BestRow<WT> o;
        o.f = __ldcg(fitc + slot);
        o.idx = slot;
#pragma unroll
        for (int w = 0; w < WT; ++w) o.r.w[w] = (w < (int)W) ? __ldcg(popc + (size_t)slot * W + w) : 0ull;
        if (better_row(o, v, W)) v = o;
    }
    return v;
}

template <int WT>
__device__ void leader_record_list(const GaArgs& a, uint32_t i, uint32_t g, uint32_t R, bool staged,
                                   const Smem& sm)
{
    record_apply<WT>(a, i, g, rec_list_best<WT>(a, i, g, R, staged, sm), R > 0, sm);
}

// Copy the ranked elites (keys rk, indices rx into generation g) to slots
// 0..E-1 of generation g+1 (R18) and publish the worst elite's key.
template <int WT>
__device__ void leader_copy_elites(const GaArgs& a, uint32_t i, uint32_t g, const uint64_t* rk, const uint32_t* rx,
                                   bool keep_ranked = false)
{
    const uint32_t W = a.ch.W, N = a.N, E = a.E;
    const uint32_t cur = g & 1u, nxt = cur ^ 1u;
    const uint64_t* popc = a.pop[cur] + (size_t)i * N * W;
    uint64_t* popn = a.pop[nxt] + (size_t)i * N * W;
    double* fitn = a.fit[nxt] + (size_t)i * a.Ns;
    // one row per thread per step: its W words are in flight together
    for (uint32_t r = threadIdx.x; r < E; r += blockDim.x) {
        Row<WT> x;
        row_load(x, popc + (size_t)rx[r] * W, W);
        row_store(x, popn + (size_t)r * W, W);
    }
    for (uint32_t r = threadIdx.x; r < E; r += blockDim.x) {
        fitn[r] = unkey(rk[r]);
        if (keep_ranked) {
            // sync point: the ranked list stays available to the export (top-K = first K) and the migrant merge
            a.rk_key[(size_t)i * kMaxElite + r] = rk[r];
            a.rk_idx[(size_t)i * kMaxElite + r] = rx[r];
        }
    }
    if (threadIdx.x == 0) a.tau[cur * a.I + i] = rk[E - 1];
}

// ------------------------------------------------------------------------
// Island exchange blocks (R16, R19): block of global island gi = xch + gi * xstride
// ------------------------------------------------------------------------
__device__ __forceinline__ uint64_t* xblock(const GaArgs& a, uint32_t gi) { return a.xch + (size_t)gi * a.xstride; }
__device__ __forceinline__ uint64_t* xrecord(const GaArgs& a, uint32_t gi)
{
    return xblock(a, gi) + (size_t)a.K * a.ch.W + a.K;
}

// leader: island i's record (cached in sm.rec) into its block
__device__ void pack_record(const GaArgs& a, uint32_t i, const Smem& sm)
{
    if (threadIdx.x == 0) {
        uint64_t* r = xrecord(a, a.island_base + i);
        const RecCache* rc = sm.rec;
        r[0] = (uint64_t)__double_as_longlong(rc->valid ? rc->f : -CUDART_INF);
        r[1] = rc->gen;
        for (uint32_t w = 0; w < a.ch.W; ++w) r[2 + w] = rc->valid ? rc->bits[w] : ~0ull;
    }
}

// leader: export island i's top-K of generation g (ranked list ix[0..K) of slots) -- rows and fitness
__device__ void export_migrants(const GaArgs& a, uint32_t i, uint32_t g, const uint32_t* ix)
{
    const uint32_t W = a.ch.W, cur = g & 1u;
    const uint64_t* pop = a.pop[cur] + (size_t)i * a.N * W;
    const double* fit = a.fit[cur] + (size_t)i * a.Ns;
    uint64_t* blk = xblock(a, a.island_base + i);
    for (uint32_t j = threadIdx.x; j < a.K * W; j += blockDim.x) {
        const uint32_t r = j / W, w = j % W;
        blk[j] = pop[(size_t)ix[r] * W + w];
    }
    for (uint32_t r = threadIdx.x; r < a.K; r += blockDim.x)
        blk[(size_t)a.K * W + r] = (uint64_t)__double_as_longlong(fit[ix[r]]);
}

// Leader, general path: the radix select already gathered the E best of
// generation g; sort them and place them.
template <int WT>
__device__ void leader_general(const GaArgs& a, uint32_t i, uint32_t g, const Smem& sm, bool keep_ranked = false)
{
    leader_sort_selected(a, i, a.E, false, sm);
    leader_copy_elites<WT>(a, i, g, sm.skey, sm.sidx, keep_ranked);
    __syncthreads();
}

// Leader, fast path of generation g.  One mbarrier gathers (TMA bulk copies)
// the per-CTA partial bests, the previous elites' fitness (slots 0..E-1 of
// generation g, ranked) and the candidate children (a superset of those that
// beat the worst previous elite).  Then: record + stall (a8), merge of the
// elites with the sorted candidates (a3), elite copy.  If the candidate list
// overflowed, the leader only stamps ctl->redo[g&1] and every CTA runs the
// general path after the barrier.
template <int WT>
__device__ void leader_fast(const GaArgs& a, uint32_t i, uint32_t g, const Smem& sm, uint32_t& mph,
                            bool keep_ranked = false)
{
    const uint32_t Ns = a.Ns, E = a.E, I = a.I, cpi = a.cpi, cpp = a.cpi_pad;
    const uint32_t cur = g & 1u, Lc = g % 3u, Lr = (g + 2u) % 3u;
    trace_mark(a, g, 0);
    if (threadIdx.x == 0) {
        // one TMA batch: record-candidate count (its 16-byte chunk) + a window of the
        // list, previous elites' fitness, candidate count chunk + a window of the list
        const uint32_t cnt_off = Lc * I + i;
        const uint32_t rwin = Ns < kRecWin ? Ns : kRecWin;
        const uint32_t b = 16u + rwin * 4u + (E > 0 ? round16(E * 8u) + cpp * 4u : 0u);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // earlier generic writes to the targets
        mbar_arrive_expect_tx(sm.mbar + 1, b);
        bulk_g2s(sm.misc + 16, a.rc_cnt + (cnt_off & ~3u), 16u, sm.mbar + 1);
        bulk_g2s(sm.rcw, a.rc_idx[Lc] + (size_t)i * Ns, rwin * 4u, sm.mbar + 1);
        if (E > 0) {
            bulk_g2s(sm.ekey, a.fit[cur] + (size_t)i * Ns, round16(E * 8u), sm.mbar + 1);
            bulk_g2s(sm.pi, a.cand_cnt + ((size_t)Lc * I + i) * cpp, cpp * 4u, sm.mbar + 1);   // per-CTA counts
        }
    }
    mbar_wait(sm.mbar + 1, mph);
    mph ^= 1u;
    if (kTrace && a.trace && threadIdx.x == 0 && blockIdx.x == 0 && g - a.g_begin < a.trace_gens)
        a.trace[(g - a.g_begin) * 16 + 15] = gtimer();
    const uint32_t R = sm.misc[16 + ((Lc * I + i) & 3u)];
    uint32_t C0 = 0;
    if (E > 0) {
        // exclusive prefix of the per-CTA candidate counts (in place), total in misc[3]
        uint32_t* cnt = sm.pi;
        if (threadIdx.x < 32) {
            uint32_t carry = 0;
            for (uint32_t c0 = 0; c0 < cpi; c0 += 32) {
                const uint32_t c = c0 + threadIdx.x;
                const uint32_t v = c < cpi ? cnt[c] : 0u;
                uint32_t incl = v;
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    const uint32_t o = __shfl_up_sync(0xFFFFFFFFu, incl, off);
                    if (threadIdx.x >= (uint32_t)off) incl += o;
                }
                if (c < cpi) cnt[c] = carry + incl - v;
                carry += __shfl_sync(0xFFFFFFFFu, incl, 31);
            }
            if (threadIdx.x == 0) { sm.misc[3] = carry; cnt[cpi] = carry; }
        }
        __syncthreads();
        C0 = sm.misc[3];
        if (C0 <= kCandCap) {
            // gather every region into skey/sidx.  Entry e of the concatenation lives in
            // region c = max{c : cnt[c] <= e}; each thread issues all of its loads (one
            // L2 round trip) before any shared-memory store.
            const uint64_t* ck = a.cand_key[Lc] + (size_t)i * cpi * a.creg;
            const uint32_t* cx = a.cand_idx[Lc] + (size_t)i * cpi * a.creg;
            constexpr uint32_t kG = (kCandCap + kBlock - 1) / kBlock;
            for (uint32_t e0 = 0; e0 < C0; e0 += kG * blockDim.x) {
                uint64_t kk[kG];
                uint32_t xx[kG];
#pragma unroll
                for (uint32_t u = 0; u < kG; ++u) {
                    const uint32_t e = e0 + u * blockDim.x + threadIdx.x;
                    if (e < C0) {
                        uint32_t lo = 0, hi = cpi - 1;
                        while (lo < hi) {
                            const uint32_t mid = (lo + hi + 1) >> 1;
                            if (cnt[mid] <= e) lo = mid; else hi = mid - 1;
                        }
                        const size_t src = (size_t)lo * a.creg + (e - cnt[lo]);
                        kk[u] = __ldcg(ck + src);
                        xx[u] = __ldcg(cx + src);
                    }
                }
#pragma unroll
                for (uint32_t u = 0; u < kG; ++u) {
                    const uint32_t e = e0 + u * blockDim.x + threadIdx.x;
                    if (e < C0) { sm.skey[e] = kk[u]; sm.sidx[e] = xx[u]; }
                }
            }
        }
        __syncthreads();
    }
    const bool ok = C0 <= kCandCap;
    // a8: record of generation g
    leader_record_list<WT>(a, i, g, R, true, sm);
    trace_mark(a, g, 1);
    if (threadIdx.x == 0) a.rc_cnt[Lr * I + i] = 0;
    if (E == 0) {
        if (threadIdx.x == 0) a.tau[cur * I + i] = ~0ull;
        return;
    }
    if (!ok) {
        if (threadIdx.x == 0) a.ctl->redo[cur] = g + 1;            // generation-stamped: no reset needed
        return;
    }
    // a3 fast path: previous elites (ranked) + candidates that beat the worst of them
    for (uint32_t r = threadIdx.x; r < E; r += blockDim.x) sm.ekey[r] = fkey(__longlong_as_double((long long)sm.ekey[r]));
    if (threadIdx.x == 0) sm.misc[2] = 0;
    __syncthreads();
    const uint64_t thr = sm.ekey[E - 1];
    for (uint32_t j0 = 0; j0 < C0; j0 += blockDim.x) {          // in-place compaction
        const uint32_t j = j0 + threadIdx.x;
        const uint64_t k = j < C0 ? sm.skey[j] : 0ull;
        const uint32_t x = j < C0 ? sm.sidx[j] : NONE;
        const bool keep = (j < C0) && k > thr;
        const unsigned m = __ballot_sync(0xFFFFFFFFu, keep);
        __syncthreads();                                            // the chunk is read before any write
        uint32_t pos = 0;
        if ((threadIdx.x & 31u) == 0 && m) pos = atomicAdd(&sm.misc[2], (uint32_t)__popc(m));
        pos = __shfl_sync(0xFFFFFFFFu, pos, 0);
        if (keep) {
            const uint32_t r = pos + __popc(m & ((1u << (threadIdx.x & 31u)) - 1u));
            sm.skey[r] = k;
            sm.sidx[r] = x;
        }
        __syncthreads();
    }
    const uint32_t C = sm.misc[2];
    const uint32_t P2 = next_pow2(C < 2 ? 2 : C);
    for (uint32_t j = C + threadIdx.x; j < P2; j += blockDim.x) { sm.skey[j] = 0ull; sm.sidx[j] = NONE; }
    bitonic_desc(sm.skey, sm.sidx, P2);
    trace_mark(a, g, 2);
    // merged rank of elite r: r + #(candidates with key > ekey[r]);
    // of candidate j: j + #(elites with key >= ckey[j])  (elites win ties: lower index)
    for (uint32_t r = threadIdx.x; r < E; r += blockDim.x) {
        const uint64_t k = sm.ekey[r];
        uint32_t lo = 0, hi = C;
        while (lo < hi) { const uint32_t mid = (lo + hi) >> 1; if (sm.skey[mid] > k) lo = mid + 1; else hi = mid; }
        const uint32_t rank = r + lo;
        if (rank < E) { sm.okey[rank] = k; sm.oidx[rank] = r; }
    }
    for (uint32_t j = threadIdx.x; j < C; j += blockDim.x) {
        const uint64_t k = sm.skey[j];
        uint32_t lo = 0, hi = E;
        while (lo < hi) { const uint32_t mid = (lo + hi) >> 1; if (sm.ekey[mid] >= k) lo = mid + 1; else hi = mid; }
        const uint32_t rank = j + lo;
        if (rank < E) { sm.okey[rank] = k; sm.oidx[rank] = sm.sidx[j]; }
    }
    __syncthreads();
    leader_copy_elites<WT>(a, i, g, sm.okey, sm.oidx, keep_ranked);
    if (threadIdx.x == 0 && i == 0) a.ctl->n_fast = ++sm.misc[8];
    trace_mark(a, g, 3);
}

// ------------------------------------------------------------------------
// Breed (a4-a7 + fused a2)
// ------------------------------------------------------------------------
template <int WT>
__device__ __forceinline__ uint32_t tournament(const GaArgs& a, uint32_t gid, uint32_t g, const double* fit,
                                               const uint4& first, const double* fpre)
{
    uint32_t best = 0;
    double bf = 0.0;
    for (uint32_t d = 0; d < a.s; d += 4) {
        const uint4 r = d == 0 ? first : philox10(make_uint4(gid, g, TAG_SELECT, d >> 2), a.key0, a.key1);
        uint32_t ids[4];
        double fs[4];
#pragma unroll
        for (int l = 0; l < 4; ++l) {
            ids[l] = below(lane_of(r, l), a.N);
            fs[l] = (d + l < a.s) ? ((d == 0 && fpre) ? fpre[l] : __ldcg(fit + ids[l])) : 0.0;
        }
#pragma unroll
        for (int l = 0; l < 4; ++l) {
            if (d + l >= a.s) break;
            if ((d + l) == 0 || fs[l] > bf || (fs[l] == bf && ids[l] < best)) { best = ids[l]; bf = fs[l]; }
        }
    }
    return best;
}

// returns the row's cut count after the repair
template <int WT>
__device__ __forceinline__ uint32_t repair(const GaArgs& a, Row<WT>& row, uint32_t gid, uint32_t g)
{
    const ChainDev& ch = a.ch;
    uint32_t c = row_popc(row, ch);
    if (c + 1 >= ch.k_min && c + 1 <= ch.k_max) return c;
    Draws dr(gid, g, TAG_REPAIR, a.key0, a.key1);
    const uint32_t npos = ch.n - 1;
    if (c > ch.k_max - 1) {
        // removals: per-word cut counts computed once, then each step finds its word by
        // a running prefix (no POPC) and clears the rr-th set bit of that word
        uint32_t cw[WT];
#pragma unroll
        for (int i = 0; i < WT; ++i) cw[i] = (uint32_t)__popcll(row.w[i]);   // no padding bits (row_popc)
        while (c > ch.k_max - 1) {
            uint32_t r = below(dr.next(), c);
            uint32_t wi = 0xFFFFFFFFu, rr = 0;
            uint64_t mw = 0;
#pragma unroll
            for (int i = 0; i < WT; ++i) {
                const bool here = (wi == 0xFFFFFFFFu) && r < cw[i];
                wi = here ? (uint32_t)i : wi;
                mw = here ? row.w[i] : mw;
                rr = here ? r : rr;
                r -= (wi == 0xFFFFFFFFu) ? cw[i] : 0u;
            }
            const uint64_t bit = 1ull << select_bit(mw, rr);
#pragma unroll
            for (int i = 0; i < WT; ++i) {
                const bool me = (uint32_t)i == wi;
                row.w[i] ^= me ? bit : 0ull;
                cw[i] -= me ? 1u : 0u;
            }
            --c;
        }
    }
    while (c < ch.k_min - 1) {                  // cuts are added only in [front_skip, n-2] (R22)
        row_toggle_rank(row, ch, below(dr.next(), npos - a.front_skip - c), false, a.front_skip);
        ++c;
    }
    return c;
}

template <int WT>
__device__ __forceinline__ void init_row(const GaArgs& a, Row<WT>& row, uint32_t gid)
{
#pragma unroll
    for (int i = 0; i < WT; ++i) row.w[i] = 0;
    Draws dr(gid, 0, TAG_INIT, a.key0, a.key1);
    const uint32_t k = a.ch.k_min + below(dr.next(), a.ch.k_max - a.ch.k_min + 1);
    const uint32_t f = a.front_skip, m = a.ch.n - 1 - f;
    for (uint32_t j = m - (k - 1); j < m; ++j) {
        const uint32_t r = below(dr.next(), j + 1);
        const uint32_t p = row_get_bit(row, f + r) ? f + j : f + r;
        row_xor_bit(row, p);
    }
}


// One child per thread.  The two children of a pair (c0 = E + 2q, c1 = c0 + 1)
// sit in adjacent lanes and swap their tournament winners with one shuffle;
// each lane then builds only its own child (R8, R18).  32-child chunks are
// dealt round-robin over every worker warp of the island (warp-major), so all
// SMs get the same share.
// Record snapshot of parity `par` of island i (f and, for narrow rows, bits)
template <int WT>
__device__ __forceinline__ BestRow<WT> load_snapshot(const GaArgs& a, uint32_t i, uint32_t par)
{
    BestRow<WT> s;
    const uint32_t sp = par * a.I + i;
    s.f = __ldcg(a.snap_f + sp);
    s.idx = 0;
#pragma unroll
    for (int w = 0; w < WT; ++w) s.r.w[w] = (WT <= 8 && w < (int)a.ch.W) ? __ldcg(a.snap_bits + (size_t)sp * a.ch.W + w) : 0ull;
    return s;
}

// Philox draws of one child for generation g (SELECT block 0, XOVER of its
// pair, MUTATE), computed ahead of the generation barrier when possible.
struct ChildDraws {
    uint4 sel, xo, mu;
};
__device__ __forceinline__ ChildDraws child_draws(const GaArgs& a, uint32_t gid, uint32_t h, uint32_t g)
{
    ChildDraws d;
    d.sel = philox10(make_uint4(gid, g, TAG_SELECT, 0), a.key0, a.key1);
    d.xo = philox10(make_uint4(gid - h, g, TAG_XOVER, 0), a.key0, a.key1);
    d.mu = philox10(make_uint4(gid, g, TAG_MUTATE, 0), a.key0, a.key1);
    return d;
}

// One child per thread.  The two children of a pair (c0 = E + 2q, c1 = c0 + 1)
// sit in adjacent lanes and swap their tournament winners with one shuffle;
// each lane then builds only its own child (R8, R18).  32-child chunks are
// dealt round-robin over every worker warp of the island (warp-major), so all
// SMs get the same share.  Candidates for the next elite merge go to this
// CTA's own region of the list (counted in shared memory, no global atomics).
template <int WT>
__device__ __forceinline__ void breed_children(const GaArgs& a, uint32_t i, uint32_t g, uint32_t wl,
                                               const uint64_t* popc, const double* fitc, uint64_t* popn,
                                               double* fitn, const uint32_t* sP, const uint32_t* sO, uint32_t spo_s,
                                               const uint64_t* tau_ptr, uint32_t* s_ccnt, uint64_t* ckey,
                                               uint32_t* cidx, uint32_t* rcnt, uint32_t* ridx,
                                               const BestRow<WT>& snap, ChildDraws& pre, bool& have_pre,
                                               const double* fpre, uint32_t* srow)
{
    const ChainDev& ch = a.ch;
    const uint32_t W = ch.W, N = a.N, E = a.E;
    const uint32_t nchild = N - E;
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    const uint32_t chunks = (nchild + 31u) / 32u;
    const uint32_t first = warp * a.cpi + wl;
    const uint64_t tau = __ldcg(tau_ptr);     // lagged elite threshold: stable during this phase
    ChildDraws nxt_dr;
    bool have_next = false;
    for (uint32_t cidx_ = first; cidx_ < chunks; cidx_ += nwarps * a.cpi) {
        const uint32_t base = cidx_ * 32u;
        const uint32_t t = base + lane;
        const bool valid = t < nchild;
        const uint32_t h = t & 1u;
        const uint32_t slot = E + t;
        const uint32_t gid = (a.island_base + i) * N + slot;
        const bool tr = kTrace && a.trace && threadIdx.x == 0 && blockIdx.x == a.I &&
                        g - a.g_begin < a.trace_gens && cidx_ == wl;
        ChildDraws dr;
        if (cidx_ == first && have_pre) dr = pre;
        else if (WT >= 8 && have_next) dr = nxt_dr;
        else dr = child_draws(a, gid, h, g);
        const uint32_t mine =
            valid ? tournament<WT>(a, gid, g, fitc, dr.sel, (cidx_ == first && have_pre) ? fpre : nullptr) : 0u;   // a4
        const uint32_t other = __shfl_xor_sync(0xFFFFFFFFu, mine, 1);
        if (tr) a.trace[(g - a.g_begin) * 16 + 8] = gtimer() + 0 * mine;
        if (!valid) continue;
        // first parent (positions < x) = own winner; second = the partner's
        Row<WT> A, B;
        row_load(A, popc + (size_t)mine * W, W);
        row_load(B, popc + (size_t)other * W, W);
        // wide rows (several chunks per warp at large N): the next chunk's Philox draws,
        // computed while this chunk's parent rows are in flight
        if constexpr (WT >= 8) {
            const uint32_t cn = cidx_ + nwarps * a.cpi;
            have_next = cn < chunks;
            if (have_next) {
                const uint32_t tn = cn * 32u + lane;
                nxt_dr = child_draws(a, (a.island_base + i) * N + E + tn, tn & 1u, g);
            }
        }
        if (tr) a.trace[(g - a.g_begin) * 16 + 9] = gtimer() + 0 * (A.w[0] ^ B.w[0]);
        if ((uint64_t)dr.xo.x < a.thr_c && ch.n >= 3) {                                   // a5
            const uint32_t x = 1 + below(dr.xo.y, ch.n - 2);
#pragma unroll
            for (int w = 0; w < WT; ++w) {
                const uint32_t lo = 64u * w;
                const uint64_t m = (x >= lo + 64) ? ~0ull : (x <= lo ? 0ull : ((1ull << (x - lo)) - 1));
                A.w[w] = (A.w[w] & m) | (B.w[w] & ~m);
            }
        }
        if (tr) a.trace[(g - a.g_begin) * 16 + 13] = gtimer() + 0 * A.w[0];
        if ((uint64_t)dr.mu.x < a.thr_m)                                                   // a6 (R22)
            row_xor_bit(A, a.front_skip + below(dr.mu.y, ch.n - 1 - a.front_skip));
        const uint32_t cuts = repair(a, A, gid, g);                                        // a7
        if (tr) a.trace[(g - a.g_begin) * 16 + 10] = gtimer() + 0 * A.w[0];
        const double f = eval_regs(ch, sP, sO, A, nullptr, srow, spo_s, cuts);             // a2
        if (tr) a.trace[(g - a.g_begin) * 16 + 11] = gtimer() + 0 * (uint64_t)__double_as_longlong(f);
        row_store(A, popn + (size_t)slot * W, W);
        fitn[slot] = f;
        append_if(fkey(f) > tau, s_ccnt, ckey, cidx, fkey(f), slot);
        if (tr) a.trace[(g - a.g_begin) * 16 + 14] = gtimer();
        // a8 filter: only children that beat a snapshot of an earlier record of this
        // island (a lower bound of the current record) can change the record
        bool improves = f > snap.f;
        if (f == snap.f) {
            if (WT > 8) {
                improves = true;                      // wide rows: the leader compares bits
            } else {
                bool decided = false;
#pragma unroll
                for (int w = WT - 1; w >= 0; --w)
                    if (w < (int)W && !decided && A.w[w] != snap.r.w[w]) { improves = A.w[w] < snap.r.w[w]; decided = true; }
            }
        }
        append_if(improves, rcnt, nullptr, ridx, 0, slot);
        if (tr) a.trace[(g - a.g_begin) * 16 + 12] = gtimer();
    }
}

// draws of this thread's first child for generation g+1 (overlaps the barrier)
__device__ __forceinline__ void precompute_draws(const GaArgs& a, uint32_t i, uint32_t g, uint32_t wl,
                                                 ChildDraws& pre, bool& have_pre)
{
    const uint32_t nchild = a.N - a.E, chunks = (nchild + 31u) / 32u;
    const uint32_t first = (threadIdx.x >> 5) * a.cpi + wl;
    have_pre = first < chunks;
    if (have_pre) {
        const uint32_t t = first * 32u + (threadIdx.x & 31u);
        pre = child_draws(a, (a.island_base + i) * a.N + a.E + t, t & 1u, g + 1);
    }
}

// sync-point phase stamps (SPLIT_TRACE builds): CTA 0 writes row `row`, slot `slot`
__device__ __forceinline__ void trace_sync(const GaArgs& a, uint32_t row, uint32_t slot)
{
    if (kTrace && a.trace && (a.export_end || row == 15) && blockIdx.x == 0 && threadIdx.x == 0 && row < a.trace_gens)
        a.trace[row * 16 + slot] = gtimer();
}

// ------------------------------------------------------------------------
// Island sync point (R16): the K worst slots of generation g (all CTAs).
// A strided fitness sample sets, per island, a threshold on the worst key
// ~fkey(f) that about kWorstCap/2 entries reach; one pass over the islands
// collects them; the leader sorts the collection (worst order: f asc, index
// desc) and keeps the first K.  The K worst are all collected whenever at
// least K entries were (every uncollected entry is better than the
// threshold), so the result is exact; when a collection holds fewer than K or
// overflows, every CTA falls back to the radix select.  Islands of at most
// kWorstSample individuals are sorted whole.
// ------------------------------------------------------------------------
template <int WT>
__device__ void select_worst(const GaArgs& a, uint32_t g, const Smem& sm, cg::grid_group& grid)
{
    const uint32_t I = a.I, N = a.N, K = a.K, cur = g & 1u;
    const bool whole = N <= kWorstSample;
    if (blockIdx.x < I) {
        const uint32_t i = blockIdx.x;
        const double* fit = a.fit[cur] + (size_t)i * a.Ns;
        const uint32_t S = whole ? N : kWorstSample;
        for (uint32_t j = threadIdx.x; j < S; j += blockDim.x) {
            const uint32_t idx = whole ? j : (uint32_t)(((uint64_t)j * N) / S);
            sm.skey[j] = ~fkey(__ldcg(fit + idx));
            sm.sidx[j] = ~idx;                          // equal fitness: the larger index is worse
        }
        __syncthreads();
        if (whole) {
            select_sorted(sm.skey, sm.sidx, S, K, sm, sm.ekey, sm.tsel);
            for (uint32_t r = threadIdx.x; r < K; r += blockDim.x) a.wslot[(size_t)i * kMaxElite + r] = ~sm.tsel[r];
        } else {
            // aim the collection at ~max(4K, 256) entries (up to 65,536 individuals: <= 512, so the
            // warp select sorts it), between K and the capacity for larger islands
            const uint64_t wide = (kWorstCap + K) / 2, narrow = 4ull * K > 256 ? 4ull * K : 256;
            const uint64_t want = (N <= 65536u && narrow < wide) ? narrow : wide;
            uint64_t pts = (want * S) / N;             // sample points at or beyond the threshold
            pts = pts < 1 ? 1 : pts;
            if (pts <= 8 && S == 16u * 128u && blockDim.x >= 512) {
                // the pts-th largest of the 2048 samples: every warp sorts its 128 and keeps its
                // top 8 (the pts-th overall is among them), one warp sorts the 16 x 8
                cta_top8_of_2048(sm.skey, sm.sidx, (uint32_t)pts, sm.okey, sm.oidx, sm.ekey, sm.tsel);
            } else {
                cta_select_sorted(sm.skey, sm.sidx, S, (uint32_t)pts, sm.hist, sm.sel, sm.misc + 4, sm.okey, sm.oidx,
                                  sm.ekey, sm.tsel);
            }
            if (threadIdx.x == 0) {
                a.wthr[i] = sm.ekey[pts - 1];           // the smallest selected key: >= pts sample points reach it
                a.wl_cnt[i] = 0;
            }
        }
    }
    if (whole) return;                                 // uniform across CTAs (N is)
    trace_sync(a, a.g_end - a.g_begin, 4);
    grid.sync();
    // one pass over the islands (I N < 2^32, checked at create): an entry at or beyond its island's
    // threshold takes a slot of the island's list with one warp-aggregated global atomic per warp,
    // island and pass step (a few hundred entries qualify in all)
    const uint32_t total = I * N, gtid = blockIdx.x * blockDim.x + threadIdx.x, gstride = gridDim.x * blockDim.x;
    uint64_t* lthr = (uint64_t*)(sm.hist + 32);        // [I] thresholds
    if (threadIdx.x < I) lthr[threadIdx.x] = __ldcg(a.wthr + threadIdx.x);
    __syncthreads();
    // eight loads in flight per thread and pass (the pass is latency-bound, not bandwidth-bound)
    constexpr uint32_t U = 8;
    const uint32_t lane = threadIdx.x & 31u;
    for (uint32_t e0 = gtid - lane; e0 < total; e0 += U * gstride) {     // warp-uniform trip count
        uint64_t wk[U];
#pragma unroll
        for (uint32_t u = 0; u < U; ++u) {
            const uint32_t e = e0 + lane + u * gstride;
            const uint32_t i = e / N;
            wk[u] = e < total ? ~fkey(__ldcg(a.fit[cur] + (size_t)i * a.Ns + (e - i * N))) : 0ull;
        }
#pragma unroll
        for (uint32_t u = 0; u < U; ++u) {
            const uint32_t e = e0 + lane + u * gstride;
            const uint32_t i = e < total ? e / N : 0u;
            const bool pass = e < total && wk[u] >= lthr[i];
            if (__any_sync(0xFFFFFFFFu, pass)) {
                const unsigned grp = __match_any_sync(0xFFFFFFFFu, pass ? i : 0xFFFFFFFFu);
                const int lead = __ffs(grp) - 1;
                uint32_t base = 0;
                if (pass && (int)lane == lead) base = atomicAdd(a.wl_cnt + i, (uint32_t)__popc(grp));
                base = __shfl_sync(0xFFFFFFFFu, base, lead);
                const uint32_t p = base + __popc(grp & ((1u << lane) - 1u));
                if (pass && p < kWorstCap) {
                    a.wl_key[(size_t)i * kWorstCap + p] = wk[u];
                    a.wl_idx[(size_t)i * kWorstCap + p] = ~(e - i * N);
                }
            }
        }
    }
    trace_sync(a, a.g_end - a.g_begin, 5);
    grid.sync();
    trace_sync(a, a.g_end - a.g_begin, 6);
    bool ok = true;
    for (uint32_t i = 0; i < I; ++i) {
        const uint32_t c = __ldcg(a.wl_cnt + i);
        ok &= (c >= K && c <= kWorstCap);
    }
    if (ok) {
        if (blockIdx.x < I) {
            const uint32_t i = blockIdx.x, C = __ldcg(a.wl_cnt + i);
            for (uint32_t j = threadIdx.x; j < C; j += blockDim.x) {
                sm.skey[j] = __ldcg(a.wl_key + (size_t)i * kWorstCap + j);
                sm.sidx[j] = __ldcg(a.wl_idx + (size_t)i * kWorstCap + j);
            }
            __syncthreads();
            select_sorted(sm.skey, sm.sidx, C, K, sm, sm.ekey, sm.tsel);
            for (uint32_t r = threadIdx.x; r < K; r += blockDim.x) a.wslot[(size_t)i * kMaxElite + r] = ~sm.tsel[r];
        }
    } else {
        general_select(a, a.fit[cur], K, true, sm, grid);
        if (blockIdx.x < I) {
            leader_sort_selected(a, blockIdx.x, K, true, sm);
            for (uint32_t r = threadIdx.x; r < K; r += blockDim.x) a.wslot[(size_t)blockIdx.x * kMaxElite + r] = sm.sidx[r];
        }
    }
}

// Leader of island i at the head of the segment after sync point g: the K best
// foreign migrants (f desc, source island asc, rank asc) replace the K worst
// slots (worst first, R16); the island record takes them in (R19); generation
// g's ranked elites are merged with them (only K slots changed: no new top-E
// selection) and placed in slots 0..E-1 of g+1 with the exact threshold.
template <int WT>
__device__ void import_migrants(const GaArgs& a, uint32_t i, uint32_t g, const Smem& sm)
{
    const uint32_t W = a.ch.W, N = a.N, E = a.E, I = a.I, cur = g & 1u;
    uint64_t* pop = a.pop[cur] + (size_t)i * N * W;
    double* fit = a.fit[cur] + (size_t)i * a.Ns;
    const uint32_t* worst_slot = a.wslot + (size_t)i * kMaxElite;
    const uint32_t gi = a.island_base + i;
    const uint32_t nf = (a.I_total - 1) * a.K;
    for (uint32_t j = threadIdx.x; j < nf; j += blockDim.x) {
        const uint32_t src = j / a.K, r = j % a.K;
        const uint32_t gsrc = src < gi ? src : src + 1;   // skip own island
        sm.skey[j] = fkey(__longlong_as_double((long long)__ldcg(xblock(a, gsrc) + (size_t)a.K * W + r)));
        sm.sidx[j] = gsrc * a.K + r;                        // ascending in (source island, rank)
    }
    __syncthreads();
    const uint32_t take = a.K < nf ? a.K : nf;
    // the K best foreign migrants in order (f desc, source asc, rank asc) -> ekey/tsel[0..take)
    select_sorted(sm.skey, sm.sidx, nf, take, sm, sm.ekey, sm.tsel);
    for (uint32_t j = threadIdx.x; j < take * W; j += blockDim.x) {
        const uint32_t r = j / W, w = j % W, e = sm.tsel[r];
        pop[(size_t)__ldcg(worst_slot + r) * W + w] = __ldcg(xblock(a, e / a.K) + (size_t)(e % a.K) * W + w);
    }
    for (uint32_t r = threadIdx.x; r < take; r += blockDim.x) fit[__ldcg(worst_slot + r)] = unkey(sm.ekey[r]);
    __syncthreads();
    // record update with the received migrants (R19)
    BestRef v{-CUDART_INF, NONE};
    for (uint32_t r = threadIdx.x; r < take; r += blockDim.x) {
        const uint32_t ws = __ldcg(worst_slot + r);
        const BestRef o{fit[ws], ws};
        if (better_rec(o.f, o.idx, v.f, v.idx, pop, W)) v = o;
    }
    v = block_best(v, pop, W, sm.scratch);
    if (threadIdx.x == 0 && v.idx != NONE) {
        bool upd = !a.rec_valid[i];
        if (!upd) upd = (v.f != a.rec_f[i]) ? (v.f > a.rec_f[i])
                                             : rows_less(pop + (size_t)v.idx * W, a.rec_bits + (size_t)i * W, W);
        if (upd) {
            a.rec_f[i] = v.f;
            a.rec_gen[i] = g;
            a.rec_valid[i] = 1;
            for (uint32_t w = 0; w < W; ++w) a.rec_bits[(size_t)i * W + w] = pop[(size_t)v.idx * W + w];
        }
    }
    if (E == 0) {
        if (threadIdx.x == 0) a.tau[cur * I + i] = ~0ull;
        return;
    }
    // migrants in ranking order (f desc, slot asc) by rank counting into skey/sidx[0..take); ranks by
    // binary search against the ranked elites (disjoint slots: K <= N - E), written to sel_* and
    // placed like any elite set
    for (uint32_t j = threadIdx.x; j < take; j += blockDim.x) sm.tsel[j] = __ldcg(worst_slot + j);
    __syncthreads();
    for (uint32_t j = threadIdx.x; j < take; j += blockDim.x) {
        const uint64_t kj = sm.ekey[j];
        const uint32_t xj = sm.tsel[j];
        uint32_t r = 0;
        for (uint32_t q = 0; q < take; ++q) r += comp_gt(sm.ekey[q], sm.tsel[q], kj, xj) ? 1u : 0u;
        sm.skey[r] = kj;
        sm.sidx[r] = xj;
    }
    __syncthreads();
    // the ranked elites into shared memory (one round trip) for the binary searches
    uint64_t* ek = sm.okey;
    uint32_t* ex = sm.oidx;
    for (uint32_t r = threadIdx.x; r < E; r += blockDim.x) {
        ek[r] = __ldcg(a.rk_key + (size_t)i * kMaxElite + r);
        ex[r] = __ldcg(a.rk_idx + (size_t)i * kMaxElite + r);
    }
    __syncthreads();
    uint64_t* ok = a.sel_key + (size_t)i * kMaxElite;
    uint32_t* ox = a.sel_idx + (size_t)i * kMaxElite;
    for (uint32_t r = threadIdx.x; r < E; r += blockDim.x) {
        const uint64_t k = ek[r];
        const uint32_t x = ex[r];
        uint32_t lo = 0, hi = take;
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (comp_gt(sm.skey[mid], sm.sidx[mid], k, x)) lo = mid + 1; else hi = mid;
        }
        if (r + lo < E) { ok[r + lo] = k; ox[r + lo] = x; }
    }
    for (uint32_t j = threadIdx.x; j < take; j += blockDim.x) {
        const uint64_t k = sm.skey[j];
        const uint32_t x = sm.sidx[j];
        uint32_t lo = 0, hi = E;
        while (lo < hi) {
            const uint32_t mid = (lo + hi) >> 1;
            if (comp_gt(ek[mid], ex[mid], k, x)) lo = mid + 1; else hi = mid;
        }
        if (j + lo < E) { ok[j + lo] = k; ox[j + lo] = x; }
    }
    __syncthreads();
    leader_copy_elites<WT>(a, i, g, ok, ox, false);
    __syncthreads();
}

// ------------------------------------------------------------------------
// The cooperative persistent GA kernel.  CTAs 0..I-1 are island leaders
// (elite selection, records); the others breed.  One grid barrier per
// generation: leader(g) runs concurrently with breed(g) because breed(g)
// needs only generation g and a lagged candidate threshold.
// ------------------------------------------------------------------------
#ifndef SPLIT_GA_MIN_BLOCKS
#define SPLIT_GA_MIN_BLOCKS 1
#endif
template <int WT>
__global__ void __launch_bounds__(kBlock, SPLIT_GA_MIN_BLOCKS) ga_kernel(GaArgs a)
{
    extern __shared__ __align__(16) uint8_t smem[];
    Smem sm;
    smem_layout(a, smem, &sm);
    cg::grid_group grid = cg::this_grid();
    stage_chain(sm.chain, a.ch, sm.mbar);
    if (a.ch.W > 4 && a.ch.W <= 16) stage_bulk(sm.po, a.ch.po, a.ch.po_bytes, sm.mbar + 2);   // (uniform)
    const uint32_t spo_s = opaque32(smem_u32(sm.po));
    const uint32_t* sP = sm.chain;
    const uint32_t* sO = sm.chain + a.ch.p_words;
    const uint32_t W = a.ch.W, N = a.N, E = a.E, I = a.I, Ns = a.Ns, cpi = a.cpi, cpp = a.cpi_pad;
    const bool is_leader = blockIdx.x < I;
    const uint32_t widx = is_leader ? 0u : blockIdx.x - I;
    const uint32_t my_island = is_leader ? NONE : widx / cpi;
    const uint32_t my_local = widx % cpi;
    const bool worker = !is_leader && my_island < I;

    if (a.mode == MODE_INIT) {
        // a1: generation 0 into buffer 0 (all N individuals), partials into parity 0
        if (worker) {
            const uint32_t i = my_island;
            uint64_t* pop = a.pop[0] + (size_t)i * N * W;
            double* fit = a.fit[0] + (size_t)i * Ns;
            BestRow<WT> best;
            best.f = -CUDART_INF;
            best.idx = NONE;
            const uint32_t warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5, chunks = (N + 31u) / 32u;
            for (uint32_t cc = warp * cpi + my_local; cc < chunks; cc += nwarps * cpi) {
                const uint32_t c = cc * 32u + (threadIdx.x & 31u);
                if (c >= N) continue;
                Row<WT> r;
                init_row(a, r, (a.island_base + i) * N + c);
                const double f = eval_regs(a.ch, sP, sO, r, nullptr, sm.rows + threadIdx.x * (2 * W + 1), spo_s);
                row_store(r, pop + (size_t)c * W, W);
                fit[c] = f;
                track_row(best, f, c, r, W);
            }
            best = block_best_row(best, W, (BestRow<WT>*)sm.scratch);
            if (threadIdx.x == 0) write_partial(a, (size_t)i * cpp + my_local, best, W);
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            a.ctl->full = 1;
            a.ctl->done = 0;
            a.ctl->gens_run = 0;
            a.ctl->n_general = 0;
            a.ctl->n_fast = 0;
            a.ctl->redo[0] = 0;
            a.ctl->redo[1] = 0;
        }
        grid.sync();
        if (is_leader) {
            rec_load(a, blockIdx.x, sm);
            leader_record<WT>(a, blockIdx.x, 0, 0, sm);
            pack_record(a, blockIdx.x, sm);
        }
        return;
    }

    // MODE_RUN: generations [g_begin, g_end).  Candidate lists rotate mod 3:
    // list g%3 holds the candidates of generation g (consumed by leader(g)),
    // breed(g) appends generation g+1's to list (g+1)%3, leader(g) resets (g+2)%3.
    if (__ldcg(&a.ctl->done)) return;            // islands: the stall rule stopped the run at a sync point
    if (a.after_import) {
        // sync point g = g_begin, after the all-gather of the exchange blocks: the global record and
        // the stall rule (R11, R19) -- decided by CTA 0 from the gathered records, identical on every
        // rank, followed by every CTA -- then the migrant import (leaders), then breeding
        const uint32_t g = a.g_begin;
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            double gf = -CUDART_INF;
            for (uint32_t gi = 0; gi < a.I_total; ++gi)
                gf = fmax(gf, __longlong_as_double((long long)__ldcg(xrecord(a, gi))));
            if (gf > a.ctl->gf_improve) {
                a.ctl->gf_improve = gf;
                a.ctl->g_last_improve = g;
            }
            if (a.stall > 0 && g - a.ctl->g_last_improve >= a.stall) {
                a.ctl->done = 1;
                a.ctl->gens_run = g;
            }
        }
        trace_sync(a, 15, 0);
        grid.sync();
        trace_sync(a, 15, 1);
        if (__ldcg(&a.ctl->done)) return;
        if (is_leader) import_migrants<WT>(a, blockIdx.x, g, sm);
        trace_sync(a, 15, 2);
        grid.sync();
        trace_sync(a, 15, 3);
    }
    if (a.init_gstall && blockIdx.x == 0 && threadIdx.x == 0) {
        // global record of generation 0 from the gathered records (read before any block is rewritten:
        // leaders pack their records only in the segment's tail, after at least one grid barrier)
        double gf = -CUDART_INF;
        for (uint32_t gi = 0; gi < a.I_total; ++gi)
            gf = fmax(gf, __longlong_as_double((long long)__ldcg(xrecord(a, gi))));
        a.ctl->gf_improve = gf;
        a.ctl->g_last_improve = 0;
    }
    const bool first_full = __ldcg(&a.ctl->full) != 0;
    uint32_t mph = 0;
    ChildDraws pre;
    bool have_pre = false;
    double fpre[4];                   // prefetched fitness of the first tournament (s <= 4)
    bool have_fpre = false;
    // generation barrier: a monotonic counter; this launch starts where the previous one left it
    // (ctl->gbar_base is written only after the last arrival of a launch, so every CTA reads the
    // same base before any arrival of this one)
    unsigned int bar_target = __ldcg(&a.ctl->gbar_base);
    BestRow<WT> snap;
    snap.f = -CUDART_INF;         // first phase of a launch: no filter (all children compared)
    snap.idx = 0;
#pragma unroll
    for (int w = 0; w < WT; ++w) snap.r.w[w] = ~0ull;
    if (worker) snap = load_snapshot<WT>(a, my_island, (a.g_begin + 1u) & 1u);   // REC(g_begin - 1), or INIT
    if (threadIdx.x == 0) sm.misc[24] = 0;
    __syncthreads();
    if (is_leader) {
        rec_load(a, blockIdx.x, sm);
        if (threadIdx.x == 0) {
            mbar_init(sm.mbar + 1, 1);
            sm.misc[8] = __ldcg(&a.ctl->n_fast);
            sm.misc[9] = __ldcg(&a.ctl->n_general);
        }
        __syncthreads();
    }
    uint32_t g = a.g_begin;
    for (; g < a.g_end; ++g) {
        const uint32_t cur = g & 1u, nxt = cur ^ 1u;
        const uint32_t Lb = (g + 1u) % 3u;
        uint32_t tau_par = nxt;               // fast path: worst elite of generation g-1 (lagged)
        if (g == a.g_begin && a.after_import) {
            tau_par = cur;                    // the import placed generation g's elites (exact threshold)
        } else if (g == a.g_begin && first_full && E > 0) {
            // generation 0 or just after migration: exact top-E first, then breed
            general_select(a, a.fit[cur], E, false, sm, grid);
            if (is_leader) {
                // the record of generation g_begin was taken by INIT or at the end of
                // the previous segment (and by the migrant import)
                leader_general<WT>(a, blockIdx.x, g, sm);
                if (threadIdx.x == 0) {
                    a.rc_cnt[((g + 2u) % 3u) * I + blockIdx.x] = 0;
                    if (blockIdx.x == 0) a.ctl->n_general = ++sm.misc[9];
                }
            }
            grid.sync();
            if (__ldcg(&a.ctl->done)) break;
            tau_par = cur;                    // exact threshold of generation g
        } else if (is_leader) {
            leader_fast<WT>(a, blockIdx.x, g, sm, mph);
        }
        if (worker) {
            // a4-a7 + a2: children of generation g+1
            const uint32_t i = my_island;
            if (kTrace && threadIdx.x == 0 && blockIdx.x == I && a.trace && g - a.g_begin < a.trace_gens)
                a.trace[(g - a.g_begin) * 16 + 4] = gtimer();
            const size_t reg = ((size_t)i * cpi + my_local) * a.creg;    // this CTA's candidate region
            breed_children<WT>(a, i, g, my_local, a.pop[cur] + (size_t)i * N * W, a.fit[cur] + (size_t)i * Ns,
                               a.pop[nxt] + (size_t)i * N * W, a.fit[nxt] + (size_t)i * Ns, sP, sO, spo_s,
                               a.tau + tau_par * I + i, sm.misc + 24, a.cand_key[Lb] + reg, a.cand_idx[Lb] + reg,
                               a.rc_cnt + Lb * I + i, a.rc_idx[Lb] + (size_t)i * Ns, snap, pre, have_pre,
                               have_fpre ? fpre : nullptr, sm.rows + threadIdx.x * (2 * W + 1));
            snap = load_snapshot<WT>(a, i, nxt);
            if (kTrace && threadIdx.x == 0 && blockIdx.x == I && a.trace && g - a.g_begin < a.trace_gens)
                a.trace[(g - a.g_begin) * 16 + 5] = gtimer();
        }
        // arrive: the CTA barrier of the arrival also orders this CTA's candidate
        // appends before thread 0 publishes their count (released with the arrival)
        __syncthreads();
        if (threadIdx.x == 0) {
            if (worker) {
                a.cand_cnt[((size_t)Lb * I + my_island) * cpp + my_local] = sm.misc[24];
                sm.misc[24] = 0;
            }
            if (kTrace && a.trace && g - a.g_begin >= 40 && g - a.g_begin < 40 + kTraceArrGens)
                a.trace[a.trace_gens * 16 + (g - a.g_begin - 40) * 1024 + blockIdx.x] = gtimer();
            asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(a.gbar) : "memory");
        }
        if (worker) precompute_draws(a, my_island, g, my_local, pre, have_pre);
        bar_target += gridDim.x;
        gbar_wait(a.gbar, bar_target);
        if (kTrace && threadIdx.x == 0 && a.trace && g - a.g_begin < a.trace_gens) {
            if (blockIdx.x == 0) a.trace[(g - a.g_begin) * 16 + 6] = gtimer();
            if (blockIdx.x == I) a.trace[(g - a.g_begin) * 16 + 7] = gtimer();
        }
        if (g == a.g_begin && blockIdx.x == 0 && threadIdx.x == 0) a.ctl->full = 0;   // every CTA read it earlier
        // one L2 round trip after the barrier: the stop / redo flags and the first
        // tournament's fitness gathers of generation g+1 are issued together
        have_fpre = false;
        if (worker && have_pre && a.s <= 4) {
            const double* fitq = a.fit[nxt] + (size_t)my_island * Ns;
#pragma unroll
            for (uint32_t l = 0; l < 4; ++l) fpre[l] = (l < a.s) ? __ldcg(fitq + below(lane_of(pre.sel, l), N)) : 0.0;
            have_fpre = true;
        }
        const uint32_t done_f = __ldcg(&a.ctl->done);
        const uint32_t redo_f = __ldcg(&a.ctl->redo[cur]);
        if (done_f) break;
        if (redo_f == g + 1) {
            have_fpre = false;                // the exact top-E rewrites elite slots of g+1
            // a candidate list overflowed: exact top-E of generation g (still intact)
            general_select(a, a.fit[cur], E, false, sm, grid);
            if (is_leader) {
                leader_general<WT>(a, blockIdx.x, g, sm);
                if (threadIdx.x == 0 && blockIdx.x == 0) a.ctl->n_general = ++sm.misc[9];
            }
            grid.sync();
        }
    }
    if (g == a.g_end) {
        trace_sync(a, a.g_end - a.g_begin, 0);
        if (a.export_end && E > 0) {
            // sync point: generation g's elite step now (record + candidate merge, or the exact radix
            // path after an overflow); the import merges the migrants into its ranked list
            if (is_leader) leader_fast<WT>(a, blockIdx.x, g, sm, mph, true);
            trace_sync(a, a.g_end - a.g_begin, 1);
            grid.sync();
            trace_sync(a, a.g_end - a.g_begin, 2);
            if (__ldcg(&a.ctl->redo[g & 1u]) == g + 1) {
                general_select(a, a.fit[g & 1u], E, false, sm, grid);
                if (is_leader) leader_general<WT>(a, blockIdx.x, g, sm, true);
            }
        } else if (is_leader) {
            // record (and stall) of the last generation of the segment
            const uint32_t R = __ldcg(a.rc_cnt + (g % 3u) * I + blockIdx.x);
            leader_record_list<WT>(a, blockIdx.x, g, R, false, sm);
        }
        if (a.export_end) {
            if (E > 0 && a.K <= E) {
                if (is_leader) {
                    __syncthreads();
                    export_migrants(a, blockIdx.x, g, a.rk_idx + (size_t)blockIdx.x * kMaxElite);   // top-K = first K
                }
            } else {
                // K > E (or E = 0): the island's top-K by the radix select
                general_select(a, a.fit[g & 1u], a.K, false, sm, grid);
                if (is_leader) {
                    leader_sort_selected(a, blockIdx.x, a.K, false, sm);
                    export_migrants(a, blockIdx.x, g, sm.sidx);
                }
            }
        }
        trace_sync(a, a.g_end - a.g_begin, 3);
        if (a.export_end) select_worst<WT>(a, g, sm, grid);
        trace_sync(a, a.g_end - a.g_begin, 7);
        if (is_leader) pack_record(a, blockIdx.x, sm);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        a.ctl->gens_run = g;
        a.ctl->gbar_base = bar_target;
    }
}

// ------------------------------------------------------------------------
// Launchers
// ------------------------------------------------------------------------
size_t ga_smem_bytes(const GaArgs& a) { return smem_layout(a, nullptr, nullptr); }

template <int WT>
static void* ga_fn()
{
    return (void*)ga_kernel<WT>;
}

static void* ga_pick(uint32_t W)
{
    if (W <= 1) return ga_fn<1>();
    if (W <= 2) return ga_fn<2>();
    if (W <= 4) return ga_fn<4>();
    if (W <= 8) return ga_fn<8>();
    if (W <= 16) return ga_fn<16>();
    return ga_fn<64>();
}

int ga_max_blocks_per_sm(uint32_t W)
{
    (void)W;
    return SPLIT_GA_MIN_BLOCKS;
}

int ga_grid(const GaArgs& a, int num_sms, cudaError_t* err)
{
    void* fn = ga_pick(a.ch.W);
    const size_t sm = ga_smem_bytes(a);
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int per_sm = 0;
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, kBlock, sm);
    if (err) *err = e;
    if (e != cudaSuccess || per_sm < 1) return 0;
    return per_sm * num_sms;
}

cudaError_t launch_ga(const GaArgs& a, int grid, cudaStream_t st, uint64_t* launches)
{
    cudaError_t e;
    if (grid < 2 * (int)a.I) return cudaErrorInvalidConfiguration;
    void* fn = ga_pick(a.ch.W);
    GaArgs copy = a;
    void* args[] = {&copy};
    e = cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kBlock), args, ga_smem_bytes(a), st);
    if (launches) ++*launches;
    return e;
}

}  // namespace splitga
