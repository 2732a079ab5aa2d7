// split_internal.h — device state and kernel launchers shared by split_host.cpp
// and the kernel units split_eval.cu / split_ga.cu (product code; nothing here is shared with oracle/).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace splitga {

constexpr uint32_t kMaxLocalIslands = 16;   // islands batched on one device
constexpr uint32_t kMaxElite = 1024;        // E and K (v1 bound)
constexpr uint32_t kCandCap = 2048;         // fast elite merge handles up to this many candidates
constexpr uint32_t kRecWin = 256;           // record-candidate entries staged by TMA
constexpr uint32_t kMaxWords = 64;          // n_ops <= 4097
constexpr uint32_t kTraceArrGens = 8;       // SPLIT_TRACE: generations whose per-CTA arrivals are kept
constexpr uint32_t kBlock = 512;            // threads per CTA of the GA kernel (one CTA per SM)

enum Tag : uint32_t { TAG_INIT = 1, TAG_SELECT = 2, TAG_XOVER = 3, TAG_MUTATE = 4, TAG_REPAIR = 5 };
enum Mode : uint32_t { MODE_INIT = 0, MODE_RUN = 1 };
constexpr uint32_t kWorstCap = 2048;        // worst-slot candidates collected per island at a sync point
constexpr uint32_t kWorstSample = 2048;     // fitness sample that sets the collection threshold

// device-resident control block (one per handle)
struct Ctl {
    uint32_t full;          // next SEL must use the general (radix) top-E path
    uint32_t done;          // stall reached (single island, in-kernel)
    uint32_t gens_run;      // generation reached by the last RUN segment
    uint32_t last_improve;  // generation of the last strict improvement (single island)
    double f_improve;       // record fitness at the last improvement
    uint32_t n_general, n_fast;
    uint32_t redo[2];       // redo[g&1] == g+1: a leader's candidate list overflowed in generation g
    double gf_improve;      // islands: global record at the last strict improvement (sync points, R11)
    uint32_t g_last_improve;
    uint32_t gbar_base;     // generation-barrier count reached by the last RUN launch (monotonic)
};

// Chain staged for the kernels: P[0..n] (u32, exclusive prefix of the latencies)
// padded to a multiple of 4 words, then ovh[0..n-2] (u32) padded likewise.
struct ChainDev {
    const uint32_t* words;  // device
    uint32_t n, W;
    uint32_t p_words, o_words;  // padded lengths (multiples of 4)
    uint32_t T;                 // == P[n]
    uint32_t k_min, k_max;
    uint64_t last_mask;         // valid bits of word W-1
    const uint2* po;            // device: po[p] = {P[p+1], ovh[p]}, p in [0, n-2] (padded)
    uint32_t po_bytes;          // multiple of 16
    // correctly rounded reciprocals for Eq. 2's divisions (split_device.cuh div_rcp_rn):
    // rcp[0] = RN(1/T), rcp[k] = RN(1/k) and rcp[n + 1 + k] = RN(1/(k T)) for k in [1, n]
    const double* rcp;          // device, 2n + 2 entries
};

// All device pointers and scalars the GA kernel needs (passed by value).
struct GaArgs {
    ChainDev ch;
    uint32_t N, E, s, K;               // population, elites, tournament size, migrants
    uint32_t I, island_base, I_total;  // local islands, first global island, all islands
    uint32_t front_skip, stall;
    uint64_t thr_c, thr_m;             // Bernoulli thresholds floor(p * 2^32)
    uint32_t key0, key1;               // Philox key (seed lo, hi)
    uint32_t mode, g_begin, g_end;     // MODE_*, generation range of a RUN segment
    uint32_t stall_in_kernel;          // single global island: stall checked every generation
    uint32_t sort_cap;                 // power of two, entries the leader can sort in smem
    uint32_t Ns;                       // island stride of fit/cand arrays (N rounded up to 4)
    uint32_t cpi, cpi_pad;             // worker CTAs per island; partial-array stride (mult. of 4)
    uint32_t stage_bits;               // leader stages partial bits in smem (small W)
    uint64_t* pop[2];                  // [I][N][W]
    double* fit[2];                    // [I][Ns]
    uint64_t* cand_key[3];             // [I][cpi][creg] candidates of generation g (list g%3),
    uint32_t* cand_idx[3];             //   one region per worker CTA
    uint32_t* cand_cnt;                // [3][I][cpi_pad] per-CTA candidate counts
    uint32_t creg;                     // region size per worker CTA
    uint64_t* sel_key;                 // [I][kMaxElite] general-select / elite output
    uint32_t* sel_idx;
    uint32_t* sel_cnt;                 // [I]
    uint64_t* tau;                     // [2][I] key of the worst elite of generation g (parity g&1)
    uint32_t* ghist;                   // [3][I][256]
    double* part_f;                    // [2][I][cpi_pad] per-CTA best child
    uint32_t* part_idx;
    uint64_t* part_bits;               // [2][I][cpi_pad][W] bits of each per-CTA best
    double* rec_f;                     // [I] island records
    uint64_t* rec_bits;                // [I][W]
    uint32_t* rec_gen;                 // [I]
    uint32_t* rec_valid;               // [I]
    // exchange blocks, one per GLOBAL island (all-gathered in one NCCL call at a sync point):
    // [K][W] migrant rows | [K] migrant fitness (f64 bits) | record: f64 bits, generation, [W] bits
    uint64_t* xch;
    uint32_t xstride;                  // words per block: K W + K + 2 + W
    uint32_t export_end;               // RUN: the segment ends at a sync point: elites, export, record
    uint32_t after_import;             // RUN: generation g_begin's elites were placed by the import
    uint32_t init_gstall;              // RUN: set the global stall state from the gathered gen-0 records
    uint64_t* rk_key;                  // [I][kMaxElite] ranked elites of the last elite step (f keys)
    uint32_t* rk_idx;                  //   and their slots
    uint32_t* wslot;                   // [I][kMaxElite] the K worst slots (worst first) at the sync point
    uint64_t* wthr;                    // [I] collection threshold on the worst key ~fkey(f)
    uint64_t* wl_key;                  // [I][kWorstCap] collected (worst key, ~slot) candidates
    uint32_t* wl_idx;
    uint32_t* wl_cnt;                  // [I]
    uint32_t* rc_cnt;                  // [3][I] record-candidate lists (children that beat a
    uint32_t* rc_idx[3];               //        snapshot of the island record), rotation as cand_*
    double* snap_f;                    // [2][I] record snapshots (parity g&1), read by breed(g+1)
    uint64_t* snap_bits;               // [2][I][W]
    Ctl* ctl;
    unsigned int* gbar;                // generation barrier counter (RUN launches)
    unsigned long long* trace;         // optional phase timestamps (SPLIT_TRACE), [trace_gens][8]
    uint32_t trace_gens;
};

// f1 exact solvers (split_exact.cu)
enum ExhMode : int { MODE_EXH_BEST = 0, MODE_EXH_MINV = 1, MODE_EXH_ARGMIN = 2 };
constexpr uint32_t kExhThreads = 256;   // threads per CTA of the enumeration kernel
constexpr uint32_t kExhQ = 64;          // survivor queue entries per warp (>= 63)
constexpr uint32_t kExhLow = 6;         // low cut positions served by the (H, Bl) table
constexpr uint32_t kExhMaxPos = 44;     // n_ops - 1 <= 44 cut positions (2^44 splits)
struct ExhArgs {
    const uint32_t* A;     // [m+1] A[p] = P[p+1] (A[m] = T): end of a block closed by cut p
    const uint32_t* B;     // [m]   B[p] = P[p+1] - ovh[p] (mod 2^32): start offset after cut p
    void* tab;             // [(m-c+1) << c] ExhEntry
    uint32_t m, c;         // cut positions n-1, low positions
    uint32_t T, k_min, k_max;
    const double* rcp;     // ChainDev::rcp of the chain (n = m + 1)
    uint64_t outer_total;  // 2^(m-c) high-part states
    uint64_t per_thread;   // high-part states per thread
    void* res;             // [grid] per-CTA best (MODE_EXH_BEST)
    const uint64_t* kv;    // [k_max+1] min V per k (input of MODE_EXH_ARGMIN)
    uint64_t* kv_out;      // [k_max+1] min V (MINV) or argmin bitset (ARGMIN), atomicMin targets
    double seed_f;         // a known fitness (< 0) to seed the filter, or 0
};
size_t exh_smem_bytes(const ExhArgs& a);
int exh_blocks_per_sm(const ExhArgs& a);
// f2 QoS simulator (split_qos.cu)
constexpr uint32_t kQosThreads = 64;    // replicas per CTA (one per thread): 7 CTAs per SM fit 65,536 replicas in one wave
constexpr uint32_t kQosQueue = 32;      // pending requests a replica may hold (fast form)
constexpr uint32_t kQosQueueBig = 160;  // the re-run after an overflow (overloaded systems)
constexpr uint32_t kQosMaxAlpha = 32;
constexpr uint32_t kQosUnsplit = 0xFFFFu; // block field of a queue entry that runs unsplit (f4)
struct QosArgs {
    uint32_t n_types, n_blocks_total, n_alpha, policy;
    const uint32_t* blk_off;       // [n_types + 1] prefix of blocks per type
    const uint32_t* blk_ns;        // [n_blocks_total]
    const uint32_t* ext;           // [n_types] Ext = sum of the type's blocks
    const uint32_t* alpha_milli;   // [n_alpha]
    uint64_t n_rep;
    uint32_t n_req;
    const int64_t* arrival;        // [n_req][n_rep] (request-major)
    const uint32_t* type;          // [n_req][n_rep]
    int64_t* t_ete;                // [n_req][n_rep]
    uint32_t* viol;                // [n_rep][n_alpha]
    double* rr;                    // [n_rep][2]
    uint32_t* err;                 // 0 ok, 1 bad arrival/type, 2 queue overflow
    // f4 elastic splitting (policy 2, R23): a request arriving to >= d_max pending requests, or to >= s_max pending
    // requests of its own type, runs unsplit (one block of uns[type] ns) and joins the tail
    uint32_t d_max, s_max;
    const uint32_t* uns;           // [n_types] unsplit latency T per type (policy 2 only)
    const uint32_t* ref;           // [n_types] latency reference of violations / RR (= ext unless the caller sets it)
};
size_t qos_smem_bytes(const QosArgs& a, uint32_t qcap);
cudaError_t launch_qos(const QosArgs& a, cudaStream_t st, uint32_t qcap);

cudaError_t launch_exh_table(const ExhArgs& a, cudaStream_t st);
cudaError_t launch_exh(const ExhArgs& a, int mode, uint32_t grid, cudaStream_t st);
cudaError_t launch_exh_reduce(const void* res, uint32_t n, void* out, cudaStream_t st);
cudaError_t launch_heatmap2(const ChainDev& ch, int64_t* var_out, uint64_t* ov_out, double* fit_out, cudaStream_t st);
cudaError_t launch_dp(const uint32_t* P, const uint32_t* ovh, uint32_t n, uint32_t k_max, uint64_t* s2_out,
                      cudaStream_t st);

// Launchers (split_eval.cu, split_ga.cu).  Return cudaError_t of the launch.
cudaError_t launch_eval_batch(const ChainDev& ch, const uint64_t* bits, uint64_t n_cand, double* out,
                              cudaStream_t st, int num_sms, uint64_t* launches);
// Cooperative persistent GA kernel; grid = blocks_per_sm * num_sms.
cudaError_t launch_ga(const GaArgs& a, int grid, cudaStream_t st, uint64_t* launches);
size_t ga_smem_bytes(const GaArgs& a);
int ga_grid(const GaArgs& a, int num_sms, cudaError_t* err);
int ga_max_blocks_per_sm(uint32_t W);
cudaError_t launch_eval_stats(const ChainDev& ch, const uint64_t* bits, int64_t* stats_out /*[5]*/,
                              double* f_out, cudaStream_t st);
cudaError_t launch_selftest_philox(const uint32_t* in, uint32_t n, uint32_t* out, cudaStream_t st);
cudaError_t launch_selftest_dexp(const double* in, uint32_t n, double* out, cudaStream_t st);

}  // namespace splitga
