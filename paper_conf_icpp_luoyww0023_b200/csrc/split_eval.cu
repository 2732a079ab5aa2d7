// split_eval.cu — K1 split_eval_batch (a2) and the small self-test kernels.
// SPLIT (ICPP'23) Eq. 2 fitness over cut bitsets; see split_device.cuh for the
// shared Philox / dexp / staging helpers and DESIGN.md §5 for the design.
#include <cuda.h>
#include <stdlib.h>
#include <string.h>

#include "split_device.cuh"

namespace splitga {

// ------------------------------------------------------------------------
// K1: split_eval_batch.  Each warp stages 32 rows (coalesced 128-bit loads)
// into a padded shared tile (odd pitch: conflict-free row reads), then every
// lane walks its own candidate.
// ------------------------------------------------------------------------
constexpr int kEvalWarps = 8;

__global__ void __launch_bounds__(kEvalWarps * 32) eval_batch_kernel(ChainDev ch, const uint64_t* __restrict__ bits,
                                                                     uint64_t n_cand, double* __restrict__ out)
{
    extern __shared__ __align__(16) uint8_t smem[];
    uint32_t* s_chain = (uint32_t*)smem;
    uint64_t* mbar = (uint64_t*)(smem + (ch.p_words + ch.o_words) * 4u);
    uint64_t* s_tiles = mbar + 2;
    const uint32_t W = ch.W;
    const uint32_t pitch = W | 1u;
    stage_chain(s_chain, ch, mbar);
    const uint32_t* sP = s_chain;
    const uint32_t* sO = s_chain + ch.p_words;

    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint64_t* tile = s_tiles + (size_t)warp * 32u * pitch;
    const uint64_t n_tiles = (n_cand + 31) / 32;
    const uint64_t gw = (uint64_t)blockIdx.x * kEvalWarps + warp;
    const uint64_t nw = (uint64_t)gridDim.x * kEvalWarps;
    for (uint64_t t = gw; t < n_tiles; t += nw) {
        const uint64_t row0 = t * 32;
        const uint32_t rows = (uint32_t)((n_cand - row0) < 32 ? (n_cand - row0) : 32);
        const uint64_t* src = bits + row0 * W;
        const uint32_t nwords = rows * W;
        if (rows == 32) {
            const uint4* src4 = (const uint4*)src;        // 256*W bytes, 16-byte aligned
            const uint32_t n4 = 16u * W;
#pragma unroll 4
            for (uint32_t j = lane; j < n4; j += 32) {
                const uint4 v = __ldcs(src4 + j);
                const uint32_t w0 = 2 * j, w1 = 2 * j + 1;
                tile[(w0 / W) * pitch + (w0 % W)] = ((uint64_t)v.y << 32) | v.x;
                tile[(w1 / W) * pitch + (w1 % W)] = ((uint64_t)v.w << 32) | v.z;
            }
        } else {
            for (uint32_t j = lane; j < nwords; j += 32) tile[(j / W) * pitch + (j % W)] = __ldcs(src + j);
        }
        __syncwarp();
        if (lane < rows) {
            const uint64_t* my = tile + lane * pitch;
            const double f = eval_walk(ch, sP, sO, [&](uint32_t w) { return my[w]; }, nullptr);
            __stcs(out + row0 + lane, f);
        }
        __syncwarp();
    }
}

// K1 for W <= 16 (n_ops <= 1025).  A CTA of 256 threads streams chunks of
// kChunk = 512 rows (512*8W bytes, contiguous) into shared memory with one TMA
// bulk copy per chunk (cp.async.bulk + mbarrier), so no instructions are spent
// staging.  Per chunk:
//  1. occupancy pass: thread t builds, for rows t and t+256, the bitmask of the
//     non-empty 32-bit half-words (skewed 128-bit loads: lane l reads chunk
//     (j+l)%C at step j, conflict-free for W = 16) and masks the padding
//     positions >= n-1;
//  2. counting sort of the chunk's rows by their cut count (the number of
//     non-empty halves when W > 4: nearly every cut has its own half), with a
//     shared-memory histogram that every warp scans redundantly.  The walk's
//     trip count is a warp's maximum, so unsorted rows (k ~ U[2,32]) leave
//     about half the lanes idle; sorted groups of 32 walk nearly equal counts;
//  3. walk: warp w takes sorted group w and then group 15-w (light + heavy, so
//     the eight warps finish together) and visits each row's cuts from the
//     last one down, one iteration per cut (a predicated refill from the
//     occupancy mask when the current half is exhausted, one FLO for the bit),
//     summing the exact integer statistics; then the FP64 tail of Eq. 2;
//  4. each thread stores its row's fitness (the stores permute one 4 KB span,
//     merged in L2).
// geometry: NW warps per CTA, RPT rows per thread, NB chunk buffers
template <int W, int NW_, int RPT_, int NB_>
struct EvalCfg {
    static constexpr uint32_t H = 2 * W;                         // 32-bit halves per row
    static constexpr uint32_t NW = NW_, RPT = RPT_, NB = NB_;
    static constexpr uint32_t NT = NW * 32;                      // threads per CTA
    static constexpr uint32_t CHUNK = RPT * NT;                  // rows per chunk
    static constexpr uint32_t CHW = CHUNK * H;                   // u32 per chunk
};

// occupancy mask of one row (bit q <=> half q non-empty, padding masked)
// EXACT: the sort key is the exact cut count (one POPC per half) instead of the
// number of non-empty halves (always exact for W <= 4).
// SWZ (W = 16 only): the chunk buffer was written by a tensor TMA with the
// 128-byte swizzle -- 16-byte chunk c of row r sits at chunk c ^ (r & 7), and
// here r & 7 == lane & 7 -- so step j reads physical chunk (j + lane) & 7
// (conflict-free across each 8-lane phase) and files its nibble under the
// logical chunk.
// The half holding the last valid position (qfull, valid bits lastm) is
// captured from the registers of the pass: its padding bits are masked in the
// mask, and only a row whose padding bits are actually set writes the masked
// half back (a rare, divergent store; an unconditional read-modify-write of
// that half costs a 32-way bank conflict per warp: every lane's row has it in
// the same bank).
// min(x, 1) as one VIMNMX (the compiler otherwise emits ISETP + SEL for x != 0)
__device__ __forceinline__ uint32_t nz1(uint32_t x)
{
    uint32_t r;
    asm("min.u32 %0, %1, 1;" : "=r"(r) : "r"(x));
    return r;
}
// occupancy nibble of four halves: bit i <=> half i non-empty (adds of disjoint bits: LEAs)
__device__ __forceinline__ uint32_t nib4(const uint4& v)
{
    return nz1(v.x) + 2u * nz1(v.y) + 4u * nz1(v.z) + 8u * nz1(v.w);
}

__device__ __forceinline__ uint32_t comp4(const uint4& v, uint32_t i)
{
    return i == 0 ? v.x : (i == 1 ? v.y : (i == 2 ? v.z : v.w));
}

template <int W, bool EXACT, bool SWZ>
__device__ __forceinline__ uint32_t row_occupancy(uint32_t* my, uint32_t lane, uint32_t validocc, uint32_t qfull,
                                                  uint32_t lastm, uint32_t& cuts)
{
    constexpr uint32_t H = 2 * W;
    uint32_t occ = 0, pc = 0, vq = 0;
    uint4 ctop = make_uint4(0u, 0u, 0u, 0u);     // SWZ: logical chunk 7 (halves 28..31)
    if constexpr (SWZ) {
        // logical chunk j sits at physical chunk j ^ (lane & 7): reading in logical order is already
        // conflict-free across each 8-lane phase, and every nibble lands at a constant shift
        static_assert(W == 16, "the swizzled layout is defined for 128-byte rows");
        const uint4* my4 = (const uint4*)my;
        const uint32_t rsw = lane & 7u;
#pragma unroll
        for (uint32_t j = 0; j < 8; ++j) {
            const uint4 v = my4[j ^ rsw];
            occ += nib4(v) << (4 * j);
            if constexpr (EXACT) pc += __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
            if (j == 7) ctop = v;                // for W = 16 the padding (qfull >= 30) lives in chunk 7
        }
        vq = comp4(ctop, qfull & 3u);
        if constexpr (EXACT) {
            // padding: halves above qfull (all in chunk 7 for W = 16: qfull >= 30) and the bits of qfull >= lastm
#pragma unroll
            for (uint32_t i = 0; i < 4; ++i) {
                const uint32_t q = 28u + i;
                const uint32_t hv = comp4(ctop, i);
                pc -= (q > qfull) ? __popc(hv) : ((q == qfull && lastm) ? __popc(hv & ~lastm) : 0u);
            }
        }
    } else {
        uint32_t occr = 0;
        if constexpr (W % 2 == 0) {
            constexpr uint32_t C = W / 2;            // 16-byte chunks per row
            const uint4* my4 = (const uint4*)my;
            uint32_t cc = lane % C;
#pragma unroll
            for (uint32_t j = 0; j < C; ++j) {
                const uint4 v = my4[cc];
                if (cc == (qfull >> 2)) vq = comp4(v, qfull & 3u);
                cc = (cc + 1 == C) ? 0u : cc + 1;
                occr |= (min(v.x, 1u) | (min(v.y, 1u) << 1) | (min(v.z, 1u) << 2) | (min(v.w, 1u) << 3)) << (4 * j);
                if constexpr (W <= 4 || EXACT) pc += __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
            }
        } else {
            const uint2* my2 = (const uint2*)my;
            uint32_t cc = lane % W;
#pragma unroll
            for (uint32_t j = 0; j < W; ++j) {
                const uint2 v = my2[cc];
                if (cc == (qfull >> 1)) vq = (qfull & 1u) ? v.y : v.x;
                cc = (cc + 1 == W) ? 0u : cc + 1;
                occr |= (min(v.x, 1u) | (min(v.y, 1u) << 1)) << (2 * j);
                if constexpr (W <= 4 || EXACT) pc += __popc(v.x) + __popc(v.y);
            }
        }
        // bit 4j+i (2j+i) of occr is half 4((j+l)%C)+i: rotate into place
        const uint32_t rot = (W % 2 == 0) ? 4u * (lane % (W / 2)) : 2u * (lane % W);
        if constexpr (H == 32) occ = __funnelshift_l(occr, occr, rot);
        else occ = ((occr << rot) | (occr >> ((H - rot) % H))) & ((1u << H) - 1u);
        if constexpr (W <= 4 || EXACT) {
            // exact cut count (sort key); padding bits removed (rare halves: read back)
            for (uint32_t q = qfull + 1; q < H; ++q) pc -= __popc(my[q]);
            if (lastm) pc -= __popc(vq & ~lastm);
        }
    }
    occ &= validocc;                             // padding: positions >= n-1 live in halves >= qfull
    if (lastm) {
        const uint32_t vm = vq & lastm;
        if (vm != vq) {                          // padding bits set: mask the stored half for the walk
            const uint32_t off = SWZ ? ((qfull * 4u) ^ ((lane & 7u) << 4)) / 4u : qfull;
            my[off] = vm;
        }
        occ |= min(vm, 1u) << qfull;
    }
    cuts = (W <= 4 || EXACT) ? pc : __popc(occ);
    return occ;
}

// The walk of one row (the a2 core): visit its cuts from the last one down, one loop
// iteration per cut -- a predicated refill from the occupancy mask `occ` when the
// current half is exhausted, one FLO for the cut -- summing the exact integer
// statistics from the staged {P[p+1], ovh[p]} pairs (spo_s), then the FP64 tail of
// Eq. 2.  my_s: shared address of the row's 32-bit halves; SWZ: 128-byte swizzle
// by (r & 7).
template <bool SWZ>
__device__ __forceinline__ double walk_row(const ChainDev& ch, uint32_t occ, uint32_t my_s, uint32_t r, uint32_t spo_s)
{
    uint32_t endP = ch.T, OV = 0, cnt = 0;
    uint64_t S2 = 0;
    const uint32_t rx = SWZ ? ((r & 7u) << 4) : 0u;   // swizzle of this row's 16-byte chunks
    uint32_t v = 0, tb = spo_s;      // current half's remaining bits and chain entries (spo + 32 q)
    auto step = [&]() {
        // refill (predicated, no branch): next non-empty half when v is exhausted -- clear its
        // occupancy bit (the highest: mask below it), load it, point tb at its chain entries;
        // then take v's highest cut the same way
        const uint32_t qn = bfind32(occ);
        const bool need = (v == 0u);
        occ = need ? (occ & bmsk32(qn)) : occ;
        v = lds32_if(need, SWZ ? (my_s | ((qn << 2) ^ rx)) : my_s + 4u * qn, v);
        tb = need ? spo_s + (qn << 8) : tb;
        const uint32_t bt = bfind32(v);
        v &= bmsk32(bt);                 // clears bit bt, the highest set
        // the block after cut p runs to the previous (higher) cut and pays ovh[p] (R3)
        const uint2 e = lds64(tb + 8u * bt);
        const uint32_t tj = endP - e.x + e.y;
        S2 += (uint64_t)tj * tj;
        OV += e.y;
        endP = e.x;
    };
    // unrolled by two (no register moves between iterations)
    while (v | occ) {
        step();
        cnt += 1;
        if (!(v | occ)) break;
        step();
        cnt += 1;
    }
    const uint32_t k = cnt + 1;
    if (k < ch.k_min || k > ch.k_max) return -CUDART_INF;
    S2 += (uint64_t)endP * endP;                 // first block: ops 0 .. c_1
    const uint64_t S1 = (uint64_t)ch.T + OV;     // sum of block times = T + overheads
    const int64_t V = (int64_t)((uint64_t)k * S2 - S1 * S1);
    return eq2(k, V, OV, ch);
}

// SWZ (W = 16): every chunk -- the ragged last one included (rows past n_cand
// arrive zero-filled) -- is one or two tensor TMA copies (box: 32 halves x
// CHUNK/nbox rows, 128-byte swizzle) described by `tmap`; the chunk buffer is
// 1024-byte aligned as the swizzle requires.
template <int W, int NW_, int RPT_, int NB_, int KEY_ = 0, bool SWZ = false>
__global__ void __launch_bounds__(NW_ * 32, NW_ == 8 ? 5 : (48 / NW_ > 0 ? 48 / NW_ : 1)) eval_batch_w_kernel(ChainDev ch, const uint64_t* __restrict__ bits,
                                                                uint64_t n_cand, double* __restrict__ out,
                                                                const __grid_constant__ CUtensorMap tmap)
{
    using Cfg = EvalCfg<W, NW_, RPT_, NB_>;
    constexpr uint32_t RPT = Cfg::RPT;
    constexpr uint32_t H = Cfg::H, CHW = Cfg::CHW, NB = Cfg::NB, NT = Cfg::NT, kChunk = Cfg::CHUNK;
    constexpr uint32_t kBoxes = (kChunk + 255u) / 256u, kBoxRows = kChunk / kBoxes;
    static_assert(!SWZ || (W == 16 && kBoxRows * kBoxes == kChunk && NT % 8 == 0), "swizzled chunk geometry");
    // the chunk buffers first: the dynamic window starts 1024-byte aligned, as the 128-byte swizzle needs
    extern __shared__ __align__(1024) uint8_t smem_k1[];
    uint8_t* smem = smem_k1;
    uint32_t* s_buf = (uint32_t*)smem;                   // [NB][CHW]
    // staged chain: po[p] = {P[p+1], ovh[p]} for cut positions p in [0, n-2]
    const uint2* spo = (const uint2*)(smem + (size_t)NB * CHW * 4u);
    uint64_t* mbar = (uint64_t*)((const uint8_t*)spo + ch.po_bytes);   // [0] chain, [1], [2] chunk buffers, [3] pad
    uint32_t* s_occ = (uint32_t*)(mbar + 4);             // [kChunk] occupancy mask of each row
    uint32_t* s_hist = s_occ + kChunk;                   // [32] histogram of the sort keys
    uint16_t* s_perm = (uint16_t*)(s_hist + 32);         // [kChunk] sorted order | flags
    const uint32_t tid = threadIdx.x, lane = tid & 31u, warp = tid >> 5;
    if (tid == 0) {
        mbar_init(mbar + 1, 1);
        mbar_init(mbar + 2, 1);
    }
    if (tid < 32) s_hist[tid] = 0;
    stage_bulk((void*)spo, ch.po, ch.po_bytes, mbar);     // includes a __syncthreads
    const uint32_t npos = ch.n - 1, qfull = npos >> 5;
    const uint32_t lastm = (npos & 31u) ? ((1u << (npos & 31u)) - 1u) : 0u;
    const uint32_t validocc = (qfull >= 32u) ? ~0u : ((1u << qfull) - 1u);   // halves wholly inside [0, n-2]
    const uint32_t spo_s = opaque32(smem_u32(spo));
    const uint64_t n_chunks = (n_cand + kChunk - 1) / kChunk;
    const uint64_t n_full = SWZ ? n_chunks : n_cand / kChunk;     // chunks that go through TMA
    uint64_t c = blockIdx.x;
    auto issue = [&](uint64_t cc, uint32_t b) {
        if (tid == 0 && cc < n_full) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive_expect_tx(mbar + 1 + b, CHW * 4u);
            if constexpr (SWZ) {
#pragma unroll
                for (uint32_t x = 0; x < kBoxes; ++x) {
                    const int32_t y = (int32_t)(cc * kChunk + x * kBoxRows);
                    asm volatile(
                        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                        ::"r"(smem_u32(s_buf + b * CHW + x * kBoxRows * H)), "l"(&tmap), "r"(0), "r"(y),
                        "r"(smem_u32(mbar + 1 + b))
                        : "memory");
                }
            } else {
                bulk_g2s(s_buf + b * CHW, bits + cc * kChunk * W, CHW * 4u, mbar + 1 + b);
            }
        }
    };
    // With one buffer (W >= 12) the next chunk's TMA is issued as soon as the
    // buffer is released and the other CTAs on the SM cover the wait.
    issue(c, 0);
    uint32_t ph = 0;                             // bit b: parity of buffer b's next phase
    for (uint32_t b = 0; c < n_chunks; c += gridDim.x, b = (NB == 2) ? b ^ 1u : 0u) {
        if (NB == 2) issue(c + gridDim.x, b ^ 1u);   // buffer b^1 was released by the last barrier
        uint32_t* buf = s_buf + b * CHW;
        const uint64_t row0 = c * kChunk;
        const uint32_t rows = (uint32_t)((n_cand - row0) < kChunk ? (n_cand - row0) : kChunk);
        if (c < n_full) {
            mbar_wait(mbar + 1 + b, (ph >> b) & 1u);
            ph ^= 1u << b;
        } else {
            const uint32_t* src = (const uint32_t*)(bits + row0 * W);
            for (uint32_t e = tid; e < rows * H; e += NT) buf[e] = __ldcs(src + e);
            __syncthreads();
        }
        // 1. occupancy pass over rows tid and tid + 256
        uint32_t key[RPT], rank[RPT], flags[RPT];
        uint32_t* hist = s_hist;
#pragma unroll
        for (uint32_t h = 0; h < RPT; ++h) {
            const uint32_t row = tid + h * NT;
            key[h] = 0;
            flags[h] = 0x4000u;                  // 0x4000: no row (ragged tail), 0x8000: k out of range
            if (row < rows) {
                uint32_t cuts;
                s_occ[row] = row_occupancy<W, KEY_ != 0, SWZ>(buf + row * H, lane, validocc, qfull, lastm, cuts);
                const uint32_t ne = __popc(s_occ[row]);
                // a row with >= k_max non-empty halves (or cuts) has k > k_max
                flags[h] = (ne < ch.k_max && cuts < ch.k_max) ? 0u : 0x8000u;
                key[h] = flags[h] ? 0u : min(cuts, 31u);
            }
            // 2. counting sort by key (the histogram was zeroed after the last chunk's scan)
            rank[h] = atomicAdd(&hist[key[h]], 1u);
        }
        __syncthreads();
        {
            const uint32_t hv = hist[lane];
            uint32_t inc = hv;
#pragma unroll
            for (uint32_t o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, inc, o);
                if (lane >= o) inc += y;
            }
#pragma unroll
            for (uint32_t h = 0; h < RPT; ++h) {
                const uint32_t start = __shfl_sync(0xFFFFFFFFu, inc - hv, key[h]);
                s_perm[start + rank[h]] = (uint16_t)((tid + h * NT) | flags[h]);
            }
        }
        __syncthreads();
        if (tid < 32) s_hist[tid] = 0;           // every warp has scanned it: zero for the next chunk
        // 3. walk sorted groups w (light) and 2 NW - 1 - w (heavy)
#pragma unroll 1
        for (uint32_t h = 0; h < RPT; ++h) {
            const uint32_t grp = h ? (2u * Cfg::NW - 1u - warp) : warp;
            const uint32_t pe = s_perm[32u * grp + lane];
            const uint32_t r = pe & 0x3FFFu;
            if (pe & 0x4000u) continue;
            const double f = (pe & 0x8000u) ? -CUDART_INF
                                            : walk_row<SWZ>(ch, s_occ[r], smem_u32(buf + r * H), r, spo_s);
            __stcs(out + row0 + r, f);
        }
        __syncthreads();                         // buffer b, s_occ, s_perm released
        if (NB == 1) issue(c + gridDim.x, 0);
    }
}

// ------------------------------------------------------------------------
// K1, grouped form (W = 16): one CTA holds NG independent groups of NWG warps.
// Each group is what one CTA of eval_batch_w_kernel<16, NWG, 1, 1, 0, true>
// is -- its own swizzled chunk buffer, mbarrier, histogram and sorted order,
// synchronised by its own named barrier (bar.sync 1 + g) -- but the groups
// share one staged chain table, so an SM holds more warps and more
// independent barrier domains in the same shared memory.
// ------------------------------------------------------------------------
template <int NWG, int NG>
struct GrpCfg {
    static constexpr uint32_t CHUNK = NWG * 32, H = 32;
    static constexpr uint32_t kBoxes = (CHUNK + 255u) / 256u, kBoxRows = CHUNK / kBoxes;
    static size_t smem(uint32_t po_bytes)
    {
        return (size_t)NG * CHUNK * 128 + po_bytes + 8 * (1 + NG + 1) + (size_t)NG * (CHUNK * 6 + 128) + 64;
    }
};

__device__ __forceinline__ void named_bar(uint32_t id, uint32_t nthreads)
{
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

template <int NWG, int NG>
__global__ void __launch_bounds__(NWG * NG * 32, (48 / (NWG * NG)) > 0 ? 48 / (NWG * NG) : 1)
    eval_grp_kernel(ChainDev ch, const uint64_t* __restrict__ bits, uint64_t n_cand, double* __restrict__ out,
                    const __grid_constant__ CUtensorMap tmap)
{
    using Cfg = GrpCfg<NWG, NG>;
    constexpr uint32_t CHUNK = Cfg::CHUNK, H = Cfg::H, NTG = NWG * 32;
    static_assert(CHUNK % 8 == 0 && Cfg::kBoxRows * Cfg::kBoxes == CHUNK, "swizzled chunk geometry");
    extern __shared__ __align__(1024) uint8_t smem_grp[];
    const uint32_t tid = threadIdx.x, g = tid / NTG, gt = tid % NTG, lane = tid & 31u, gwarp = gt >> 5;
    uint32_t* buf = (uint32_t*)smem_grp + (size_t)g * CHUNK * H;          // this group's chunk buffer
    const uint2* spo = (const uint2*)(smem_grp + (size_t)NG * CHUNK * 128);
    uint64_t* mbar = (uint64_t*)((const uint8_t*)spo + ch.po_bytes);       // [0] chain, [1 + g] groups
    uint8_t* gbase = (uint8_t*)(mbar + 1 + NG + 1) + (size_t)g * (CHUNK * 6 + 128);
    uint32_t* s_occ = (uint32_t*)gbase;                                    // [CHUNK]
    uint32_t* s_hist = s_occ + CHUNK;                                      // [32]
    uint16_t* s_perm = (uint16_t*)(s_hist + 32);                           // [CHUNK]
    if (tid == 0)
        for (uint32_t q = 0; q < NG; ++q) mbar_init(mbar + 1 + q, 1);
    if (gt < 32) s_hist[gt] = 0;
    stage_bulk((void*)spo, ch.po, ch.po_bytes, mbar);                      // includes a __syncthreads
    const uint32_t npos = ch.n - 1, qfull = npos >> 5;
    const uint32_t lastm = (npos & 31u) ? ((1u << (npos & 31u)) - 1u) : 0u;
    const uint32_t validocc = (qfull >= 32u) ? ~0u : ((1u << qfull) - 1u);
    const uint32_t spo_s = opaque32(smem_u32(spo));
    const uint64_t n_chunks = (n_cand + CHUNK - 1) / CHUNK;
    const uint64_t stride = (uint64_t)gridDim.x * NG;
    uint64_t c = (uint64_t)blockIdx.x * NG + g;
    auto issue = [&](uint64_t cc) {
        if (gt == 0 && cc < n_chunks) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive_expect_tx(mbar + 1 + g, CHUNK * 128u);
#pragma unroll
            for (uint32_t x = 0; x < Cfg::kBoxes; ++x) {
                const int32_t y = (int32_t)(cc * CHUNK + x * Cfg::kBoxRows);
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                    ::"r"(smem_u32(buf + x * Cfg::kBoxRows * H)), "l"(&tmap), "r"(0), "r"(y), "r"(smem_u32(mbar + 1 + g))
                    : "memory");
            }
        }
    };
    issue(c);
    uint32_t ph = 0;
    for (; c < n_chunks; c += stride) {
        const uint64_t row0 = c * CHUNK;
        const uint32_t rows = (uint32_t)((n_cand - row0) < CHUNK ? (n_cand - row0) : CHUNK);
        mbar_wait(mbar + 1 + g, ph);
        ph ^= 1u;
        uint32_t key = 0, flags = 0x4000u;
        if (gt < rows) {
            uint32_t cuts;
            const uint32_t occ = row_occupancy<16, false, true>(buf + gt * H, lane, validocc, qfull, lastm, cuts);
            s_occ[gt] = occ;
            const uint32_t ne = __popc(occ);
            flags = (ne < ch.k_max && cuts < ch.k_max) ? 0u : 0x8000u;
            key = flags ? 0u : min(cuts, 31u);
        }
        const uint32_t rank = atomicAdd(&s_hist[key], 1u);
        named_bar(1 + g, NTG);
        {
            const uint32_t hv = s_hist[lane];
            uint32_t inc = hv;
#pragma unroll
            for (uint32_t o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, inc, o);
                if (lane >= o) inc += y;
            }
            const uint32_t start = __shfl_sync(0xFFFFFFFFu, inc - hv, key);
            s_perm[start + rank] = (uint16_t)(gt | flags);
        }
        named_bar(1 + g, NTG);
        if (gt < 32) s_hist[gt] = 0;
        {
            const uint32_t pe = s_perm[32u * gwarp + lane];
            const uint32_t r = pe & 0x3FFFu;
            if (!(pe & 0x4000u)) {
                const double f = (pe & 0x8000u) ? -CUDART_INF
                                                : walk_row<true>(ch, s_occ[r], smem_u32(buf + r * H), r, spo_s);
                __stcs(out + row0 + r, f);
            }
        }
        named_bar(1 + g, NTG);                    // this group's buffer, occupancy masks and order released
        issue(c + stride);
    }
}

// K1, grouped and double-buffered (tuning variant): like eval_grp_kernel, but each
// group owns two chunk buffers -- the next chunk's TMA is in flight while the group
// walks the current one (the single-buffered group waits for it after its
// end-of-chunk barrier).  Twice the shared memory per group: half the warps per SM.
template <int NWG, int NG>
struct Grp2Cfg {
    static constexpr uint32_t CHUNK = NWG * 32, H = 32;
    static constexpr uint32_t kBoxes = (CHUNK + 255u) / 256u, kBoxRows = CHUNK / kBoxes;
    static size_t smem(uint32_t po_bytes)
    {
        return (size_t)NG * 2 * CHUNK * 128 + po_bytes + 8 * (1 + 2 * NG + 1) + (size_t)NG * (CHUNK * 6 + 128) + 64;
    }
};

template <int NWG, int NG>
__global__ void __launch_bounds__(NWG * NG * 32, (24 / (NWG * NG)) > 0 ? 24 / (NWG * NG) : 1)
    eval_grp2_kernel(ChainDev ch, const uint64_t* __restrict__ bits, uint64_t n_cand, double* __restrict__ out,
                     const __grid_constant__ CUtensorMap tmap)
{
    using Cfg = Grp2Cfg<NWG, NG>;
    constexpr uint32_t CHUNK = Cfg::CHUNK, H = Cfg::H, NTG = NWG * 32;
    static_assert(CHUNK % 8 == 0 && Cfg::kBoxRows * Cfg::kBoxes == CHUNK, "swizzled chunk geometry");
    extern __shared__ __align__(1024) uint8_t smem_grp2[];
    const uint32_t tid = threadIdx.x, g = tid / NTG, gt = tid % NTG, lane = tid & 31u, gwarp = gt >> 5;
    uint32_t* bufs = (uint32_t*)smem_grp2 + (size_t)g * 2 * CHUNK * H;     // this group's two chunk buffers
    const uint2* spo = (const uint2*)(smem_grp2 + (size_t)NG * 2 * CHUNK * 128);
    uint64_t* mbar = (uint64_t*)((const uint8_t*)spo + ch.po_bytes);       // [0] chain, [1 + 2g + b] buffers
    uint8_t* gbase = (uint8_t*)(mbar + 1 + 2 * NG + 1) + (size_t)g * (CHUNK * 6 + 128);
    uint32_t* s_occ = (uint32_t*)gbase;
    uint32_t* s_hist = s_occ + CHUNK;
    uint16_t* s_perm = (uint16_t*)(s_hist + 32);
    if (tid == 0)
        for (uint32_t q = 0; q < 2 * NG; ++q) mbar_init(mbar + 1 + q, 1);
    if (gt < 32) s_hist[gt] = 0;
    stage_bulk((void*)spo, ch.po, ch.po_bytes, mbar);
    const uint32_t npos = ch.n - 1, qfull = npos >> 5;
    const uint32_t lastm = (npos & 31u) ? ((1u << (npos & 31u)) - 1u) : 0u;
    const uint32_t validocc = (qfull >= 32u) ? ~0u : ((1u << qfull) - 1u);
    const uint32_t spo_s = opaque32(smem_u32(spo));
    const uint64_t n_chunks = (n_cand + CHUNK - 1) / CHUNK;
    const uint64_t stride = (uint64_t)gridDim.x * NG;
    uint64_t c = (uint64_t)blockIdx.x * NG + g;
    auto issue = [&](uint64_t cc, uint32_t b) {
        if (gt == 0 && cc < n_chunks) {
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_arrive_expect_tx(mbar + 1 + 2 * g + b, CHUNK * 128u);
#pragma unroll
            for (uint32_t x = 0; x < Cfg::kBoxes; ++x) {
                const int32_t y = (int32_t)(cc * CHUNK + x * Cfg::kBoxRows);
                asm volatile(
                    "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                    ::"r"(smem_u32(bufs + b * CHUNK * H + x * Cfg::kBoxRows * H)), "l"(&tmap), "r"(0), "r"(y),
                    "r"(smem_u32(mbar + 1 + 2 * g + b))
                    : "memory");
            }
        }
    };
    issue(c, 0);
    issue(c + stride, 1);
    uint32_t ph = 0;                             // bit b: parity of buffer b's next phase
    for (uint32_t b = 0; c < n_chunks; c += stride, b ^= 1u) {
        uint32_t* buf = bufs + b * CHUNK * H;
        const uint64_t row0 = c * CHUNK;
        const uint32_t rows = (uint32_t)((n_cand - row0) < CHUNK ? (n_cand - row0) : CHUNK);
        mbar_wait(mbar + 1 + 2 * g + b, (ph >> b) & 1u);
        ph ^= 1u << b;
        uint32_t key = 0, flags = 0x4000u;
        if (gt < rows) {
            uint32_t cuts;
            const uint32_t occ = row_occupancy<16, false, true>(buf + gt * H, lane, validocc, qfull, lastm, cuts);
            s_occ[gt] = occ;
            const uint32_t ne = __popc(occ);
            flags = (ne < ch.k_max && cuts < ch.k_max) ? 0u : 0x8000u;
            key = flags ? 0u : min(cuts, 31u);
        }
        const uint32_t rank = atomicAdd(&s_hist[key], 1u);
        named_bar(1 + g, NTG);
        {
            const uint32_t hv = s_hist[lane];
            uint32_t inc = hv;
#pragma unroll
            for (uint32_t o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, inc, o);
                if (lane >= o) inc += y;
            }
            const uint32_t start = __shfl_sync(0xFFFFFFFFu, inc - hv, key);
            s_perm[start + rank] = (uint16_t)(gt | flags);
        }
        named_bar(1 + g, NTG);
        if (gt < 32) s_hist[gt] = 0;
        {
            const uint32_t pe = s_perm[32u * gwarp + lane];
            const uint32_t r = pe & 0x3FFFu;
            if (!(pe & 0x4000u)) {
                const double f = (pe & 0x8000u) ? -CUDART_INF
                                                : walk_row<true>(ch, s_occ[r], smem_u32(buf + r * H), r, spo_s);
                __stcs(out + row0 + r, f);
            }
        }
        named_bar(1 + g, NTG);                    // buffer b, occupancy masks and order released
        issue(c + 2 * stride, b);                 // buffer b takes the chunk after the one in flight
    }
}

// ------------------------------------------------------------------------
// Small kernels
// ------------------------------------------------------------------------
__global__ void eval_stats_kernel(ChainDev ch, const uint64_t* bits, int64_t* st_out, double* f_out)
{
    extern __shared__ __align__(16) uint8_t smem[];
    uint32_t* s_chain = (uint32_t*)smem;
    uint64_t* mbar = (uint64_t*)(smem + (ch.p_words + ch.o_words) * 4u);
    stage_chain(s_chain, ch, mbar);
    if (threadIdx.x == 0) {
        Stats st{};
        const double f = eval_walk(ch, s_chain, s_chain + ch.p_words, [&](uint32_t w) { return bits[w]; }, &st);
        st_out[0] = st.k; st_out[1] = st.V; st_out[2] = (int64_t)st.S1; st_out[3] = (int64_t)st.S2; st_out[4] = (int64_t)st.OV;
        *f_out = f;
    }
}

__global__ void selftest_philox_kernel(const uint32_t* in, uint32_t n, uint32_t* out)
{
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= n) return;
    const uint32_t* v = in + 6 * t;
    const uint4 r = philox10(make_uint4(v[0], v[1], v[2], v[3]), v[4], v[5]);
    out[4 * t] = r.x; out[4 * t + 1] = r.y; out[4 * t + 2] = r.z; out[4 * t + 3] = r.w;
}

__global__ void selftest_dexp_kernel(const double* in, uint32_t n, double* out)
{
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t < n) out[t] = dexp_dev(in[t]);
}

// ------------------------------------------------------------------------
// Launchers
// ------------------------------------------------------------------------
// K1 variants per row width: {kernel, warps, rows per thread, buffers}.  The
// defaults were chosen by tools/eval_sweep.py on a B200; the
// environment variable SPLIT_EVAL_VARIANT=<i> selects another (tuning only).
struct EvalVariant {
    void* fn;
    uint32_t W, NW, RPT, NB, SWZ;
    uint32_t NG = 0;                                  // grouped kernel: NG groups of NW warps per CTA
    size_t (*grp_smem)(uint32_t) = nullptr;
};

template <int NWG, int NG>
static EvalVariant eval_grp_variant()
{
    EvalVariant v{(void*)eval_grp_kernel<NWG, NG>, 16u, (uint32_t)NWG, 1u, 1u, 1u};
    v.NG = NG;
    v.grp_smem = &GrpCfg<NWG, NG>::smem;
    return v;
}
template <int NWG, int NG>
static EvalVariant eval_grp2_variant()
{
    EvalVariant v{(void*)eval_grp2_kernel<NWG, NG>, 16u, (uint32_t)NWG, 1u, 1u, 1u};
    v.NG = NG;
    v.grp_smem = &Grp2Cfg<NWG, NG>::smem;
    return v;
}

template <int W, int NW, int RPT, int NB, int KEY = 0, bool SWZ = false>
static EvalVariant eval_variant()
{
    return EvalVariant{(void*)eval_batch_w_kernel<W, NW, RPT, NB, KEY, SWZ>, (uint32_t)W, (uint32_t)NW,
                       (uint32_t)RPT, (uint32_t)NB, SWZ ? 1u : 0u};
}

static size_t eval_smem_of(const ChainDev& ch, const EvalVariant& v)
{
    const size_t chunk = (size_t)v.NW * 32 * v.RPT;
    return (size_t)ch.po_bytes + 32 + chunk * (4 + 2) + 32 * 4 + (size_t)v.NB * chunk * (2 * v.W) * 4;
}

// cuTensorMapEncodeTiled from the driver (the runtime is linked statically; the
// driver entry point needs no link-time dependency on libcuda)
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_tiled()
{
    static EncodeTiledFn fn = [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            p = nullptr;
        return (EncodeTiledFn)p;
    }();
    return fn;
}

// 2-D map over the bitsets viewed as u32 halves: [n_cand rows][32 halves], box of
// box_rows rows, 128-byte swizzle, zero fill past the last row
static bool make_row_tmap(CUtensorMap* m, const uint64_t* bits, uint64_t n_cand, uint32_t box_rows)
{
    EncodeTiledFn enc = encode_tiled();
    if (!enc) return false;
    const cuuint64_t dims[2] = {32, (cuuint64_t)n_cand};
    const cuuint64_t strides[1] = {128};
    const cuuint32_t box[2] = {32, box_rows};
    const cuuint32_t estr[2] = {1, 1};
    return enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, (void*)bits, dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int W>
static EvalVariant eval_default()
{
    if constexpr (W == 16) return eval_grp_variant<6, 4>();   // 2 CTAs x 4 groups x 6 warps per SM
    else if constexpr (W >= 12) return eval_variant<W, 15, 1, 1>();
    else if constexpr (W >= 6) return eval_variant<W, 8, 2, 1>();
    else return eval_variant<W, 8, 2, 2>();
}

static EvalVariant eval_pick(uint32_t W)
{
    static const int sel = [] {
        const char* e = getenv("SPLIT_EVAL_VARIANT");
        return e ? atoi(e) : -1;
    }();
    if (W == 16 && sel >= 0) {
        switch (sel) {
        case 100: return eval_variant<16, 15, 1, 1>();            // the round-1 default (bulk copies, no swizzle)
        case 120: return eval_variant<16, 11, 1, 1, 0, true>();   // one group per CTA, 4 CTAs x 11 warps
        case 101: return eval_variant<16, 15, 1, 1, 1, true>();
        case 102: return eval_variant<16, 16, 1, 1, 0, true>();
        case 103: return eval_variant<16, 12, 1, 1, 0, true>();
        case 104: return eval_variant<16, 8, 2, 1, 0, true>();
        case 500: return eval_grp2_variant<3, 4>();    // double-buffered groups: 2 CTAs x 4 x 3 warps per SM
        case 501: return eval_grp2_variant<6, 2>();    // 2 CTAs x 2 x 6 warps
        case 502: return eval_grp2_variant<4, 3>();    // 2 CTAs x 3 x 4 warps
        case 503: return eval_grp2_variant<2, 6>();    // 2 CTAs x 6 x 2 warps
        case 400: return eval_grp_variant<6, 4>();     // 2 CTAs x 4 groups x 6 warps per SM
        case 401: return eval_grp_variant<5, 4>();
        case 402: return eval_grp_variant<8, 3>();
        case 403: return eval_grp_variant<11, 2>();
        case 404: return eval_grp_variant<4, 6>();
        case 405: return eval_grp_variant<12, 2>();
        case 406: return eval_grp_variant<8, 2>();
        case 410: return eval_grp_variant<5, 5>();
        case 411: return eval_grp_variant<7, 3>();
        case 412: return eval_grp_variant<3, 8>();
        case 413: return eval_grp_variant<6, 3>();
        case 110: return eval_variant<16, 10, 1, 1, 0, true>();
        case 111: return eval_variant<16, 11, 1, 1, 0, true>();
        case 113: return eval_variant<16, 13, 1, 1, 0, true>();
        case 114: return eval_variant<16, 14, 1, 1, 0, true>();
        case 116: return eval_variant<16, 16, 1, 1, 0, true>();
        case 0: return eval_variant<16, 8, 1, 1>();
        case 1: return eval_variant<16, 7, 2, 1>();
        case 2: return eval_variant<16, 12, 2, 1>();
        case 3: return eval_variant<16, 4, 2, 1>();
        case 4: return eval_variant<16, 6, 2, 1>();
        case 5: return eval_variant<16, 8, 1, 2>();
        case 6: return eval_variant<16, 16, 1, 1>();
        case 7: return eval_variant<16, 15, 1, 1>();
        case 8: return eval_variant<16, 24, 1, 1>();
        case 9: return eval_variant<16, 12, 1, 1>();
        case 10: return eval_variant<16, 15, 1, 1, 1>();
        case 11: return eval_variant<16, 8, 2, 1, 1>();
        case 12: return eval_variant<16, 12, 1, 1, 1>();
        case 13: return eval_variant<16, 16, 1, 1, 1>();
        case 14: return eval_variant<16, 7, 2, 1, 1>();
        case 15: return eval_variant<16, 11, 1, 1>();
        case 16: return eval_variant<16, 9, 1, 1>();
        case 17: return eval_variant<16, 7, 1, 1>();
        case 18: return eval_variant<16, 6, 1, 1>();
        case 19: return eval_variant<16, 5, 1, 1>();
        default: break;
        }
    }
    switch (W) {
    case 1: return eval_default<1>();   case 2: return eval_default<2>();   case 3: return eval_default<3>();
    case 4: return eval_default<4>();   case 5: return eval_default<5>();   case 6: return eval_default<6>();
    case 7: return eval_default<7>();   case 8: return eval_default<8>();   case 9: return eval_default<9>();
    case 10: return eval_default<10>(); case 11: return eval_default<11>(); case 12: return eval_default<12>();
    case 13: return eval_default<13>(); case 14: return eval_default<14>(); case 15: return eval_default<15>();
    case 16: return eval_default<16>();
    default: return EvalVariant{(void*)eval_batch_kernel, W, (uint32_t)kEvalWarps, 0, 0, 0};
    }
}

cudaError_t launch_eval_batch(const ChainDev& ch, const uint64_t* bits, uint64_t n_cand, double* out, cudaStream_t st,
                              int num_sms, uint64_t* launches)
{
    if (n_cand == 0) return cudaSuccess;
    EvalVariant v = eval_pick(ch.W);
    alignas(64) CUtensorMap tmap;
    memset(&tmap, 0, sizeof(tmap));
    if (v.SWZ) {
        // tensor maps take int32 row coordinates: larger batches use the bulk-copy kernel
        const uint32_t chunk = v.NW * 32 * v.RPT, nbox = (chunk + 255) / 256;
        if (n_cand >= (1ull << 31) || !make_row_tmap(&tmap, bits, n_cand, chunk / nbox))
            v = eval_variant<16, 15, 1, 1>();
    }
    const size_t sm = v.NG ? v.grp_smem(ch.po_bytes)
                           : v.RPT ? eval_smem_of(ch, v)
                                   : (size_t)(ch.p_words + ch.o_words) * 4 + 16 + (size_t)kEvalWarps * 32 * (ch.W | 1u) * 8;
    cudaError_t e = cudaFuncSetAttribute(v.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    const uint32_t nt = 32u * v.NW * (v.NG ? v.NG : 1u);
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, v.fn, (int)nt, sm);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) per_sm = 1;
    const uint64_t rows_per_cta = v.RPT ? (uint64_t)nt * v.RPT : nt;
    uint64_t grid = (uint64_t)per_sm * num_sms;
    const uint64_t need = (n_cand + rows_per_cta - 1) / rows_per_cta;
    if (grid > need) grid = need;
    ChainDev c = ch;
    const uint64_t* b = bits;
    double* o = out;
    void* args[] = {&c, &b, &n_cand, &o, &tmap};
    e = cudaLaunchKernel(v.fn, dim3((unsigned)grid), dim3(nt), args, sm, st);
    if (launches) ++*launches;
    return e;
}

cudaError_t launch_eval_stats(const ChainDev& ch, const uint64_t* bits, int64_t* stats_out, double* f_out,
                              cudaStream_t st)
{
    const size_t sm = (size_t)(ch.p_words + ch.o_words) * 4 + 16;
    cudaError_t e = cudaFuncSetAttribute(eval_stats_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    eval_stats_kernel<<<1, 32, sm, st>>>(ch, bits, stats_out, f_out);
    return cudaGetLastError();
}

cudaError_t launch_selftest_philox(const uint32_t* in, uint32_t n, uint32_t* out, cudaStream_t st)
{
    if (n == 0) return cudaSuccess;
    selftest_philox_kernel<<<(n + 127) / 128, 128, 0, st>>>(in, n, out);
    return cudaGetLastError();
}

cudaError_t launch_selftest_dexp(const double* in, uint32_t n, double* out, cudaStream_t st)
{
    if (n == 0) return cudaSuccess;
    selftest_dexp_kernel<<<(n + 127) / 128, 128, 0, st>>>(in, n, out);
    return cudaGetLastError();
}

}  // namespace splitga
