/*
 * split_ga.h — C ABI of the B200 GA split search (SPLIT, ICPP'23, §3.3).
 *
 * The library searches for "evenly-sized" splits of a model's operator chain:
 * m-1 cut points divide the model into m blocks (PAPER.md P@20780-20831) and a
 * genetic algorithm maximises Eq. 2 (P@21101-21296)
 *
 *     fitness = -( e^(sigma/T - 1) + e^(overhead/m - 1) )
 *
 * where sigma is the (population) standard deviation of the block execution
 * times, T the vanilla model's execution time and overhead the splitting
 * overhead ratio (fn. 2, P@13393-13520).  The GA steps follow P@21534-22160;
 * every detail the paper leaves open is fixed by the readings R1-R19 of
 * DESIGN.md §3.  Algorithm 1 (greedy preemption, P@27209-28515) is exposed as
 * a host-only decision function.
 *
 * Conventions
 *  - Every entry point returns an int status: SPLIT_OK (0) or a negative
 *    SPLIT_E_* code; split_strerror() names it and split_last_error() gives a
 *    thread-local detail string.  Nothing is thrown across the ABI.
 *  - Device work runs on the handle's stream (params.stream, a cudaStream_t;
 *    NULL = the legacy default stream) and device params.device.
 *  - Bitset layout: candidate c is row c of a dense row-major uint64_t[N][W],
 *    W = ceil((n_ops-1)/64) words (split_words()).  Bit p of the row (word
 *    p>>6, bit p&63) means "cut between operator p and operator p+1",
 *    p in [0, n_ops-2].  Bits >= n_ops-1 in the last word are padding: ignored.
 *  - Integer-ns latencies; block times, S1 = sum t, S2 = sum t^2 and
 *    V = k*S2 - S1^2 (= k^2 sigma^2) are exact integers; the FP64 tail
 *    follows DESIGN.md R5'/R5'' so results are bit-reproducible.
 *  - A handle is not thread-safe; distinct handles are independent.
 */
#ifndef SPLIT_GA_H
#define SPLIT_GA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
    SPLIT_OK = 0,
    SPLIT_E_INVAL = -1,  /* null pointer, zero size, out-of-range parameter   */
    SPLIT_E_RANGE = -2,  /* latency/overhead magnitudes break the int guards  */
    SPLIT_E_ALIGN = -3,  /* device buffer not 16-byte (bits) / 8-byte aligned */
    SPLIT_E_NOMEM = -4,  /* device or host allocation failed                  */
    SPLIT_E_CUDA = -5,   /* CUDA runtime error (see split_last_error)         */
    SPLIT_E_NCCL = -6,   /* NCCL error or NCCL not loadable                   */
    SPLIT_E_STATE = -7   /* call not valid in the handle's state              */
};

typedef struct split_ga_t split_ga_t;  /* opaque; owns device state */

/* GA parameters.  Paper-silent choices and their defaults: DESIGN.md R6-R11,
 * R16-R18.  split_ga_params_default() fills every field. */
typedef struct {
    uint32_t pop_size;          /* N individuals per island, >= 2                        */
    uint32_t n_elite;           /* E, 0..min(N,1024); (N - E) must be even  (P@21965-22054) */
    uint32_t tournament_size;   /* s, 1..32                                  (R7)        */
    double p_crossover;         /* [0,1]  one-point crossover probability    (P@21745-21902) */
    double p_mutation;          /* [0,1]  per-child one-bit-flip probability (P@21906-21963) */
    uint32_t k_min, k_max;      /* block-count range, 1 <= k_min <= k_max <= n_ops (R6)  */
    uint32_t front_skip;        /* every cut the GA places (init, mutation, repair) lies in
                                   [front_skip, n_ops-2] (observation "far from the
                                   front", P@19225-19437; R22)               */
    uint32_t stall_generations; /* stop after this many generations without a strictly
                                   better fitness; 0 = off               (P@22056-22160) */
    const int64_t* cut_overhead_ns; /* host, n_ops-1 entries: extra time the block after
                                   cut p pays (R3); NULL = all 0.  Copied at create.     */
    uint32_t island_id;         /* first global island this handle runs                 */
    uint32_t n_islands;         /* total islands across all ranks                       */
    uint32_t islands_per_device;/* islands this handle runs: [island_id, +islands_per_device) */
    uint32_t migration_interval;/* M: migrate every M generations (0 = off)     (R16)   */
    uint32_t n_migrants;        /* K: migrants per island, 1 <= K <= N - E when M > 0    */
    void* comm;                 /* split_comm_init() communicator when islands span ranks,
                                   NULL when every island is on this device              */
    int device;                 /* CUDA device ordinal                                   */
    void* stream;               /* cudaStream_t for all device work (NULL = default)     */
} split_ga_params;

void split_ga_params_default(split_ga_params* p);

/* a0 — validate and stage a chain.  latencies_ns: host, n_ops >= 2 entries,
 * each >= 0, sum T >= 1.  Computes the exclusive prefix P[0..n], copies
 * P and the overheads to the device (u32), sets the Bernoulli thresholds and
 * allocates the population for islands_per_device islands.
 * Guards (SPLIT_E_RANGE): T' = T + (sum of the k_max-1 largest overheads) must
 * be < 2^32 and (k_max-1)*T'^2 < 2^63 so every segment sum fits u32, S2 fits
 * u64 and V fits int64.  *out is set only on success. */
int split_ga_create(const int64_t* latencies_ns, uint32_t n_ops, const split_ga_params* p,
                    split_ga_t** out);

uint32_t split_words(const split_ga_t* h);  /* W = ceil((n_ops-1)/64); 0 on NULL */

/* a2 — score candidates with Eq. 2.  cut_bitsets: DEVICE pointer to n_cand*W
 * words, 16-byte aligned (SPLIT_E_ALIGN); fitness_out: DEVICE pointer to n_cand
 * doubles, 8-byte aligned.  Candidates with k outside [k_min, k_max] get
 * -INFINITY.  Asynchronous on the handle's stream; buffers are caller-owned and
 * must live until the stream work completes.  n_cand = 0 is a no-op. */
int split_eval_batch(split_ga_t* h, const uint64_t* cut_bitsets, uint64_t n_cand, double* fitness_out);

/* a2 through HOST buffers: copies the bitsets in, evaluates and copies the
 * fitness back in chunks, overlapping copies with compute.  Synchronous.  Any
 * host pointers are accepted; page-locked ones are fastest. */
int split_eval_batch_host(split_ga_t* h, const uint64_t* cut_bitsets_host, uint64_t n_cand,
                          double* fitness_out_host);

/* Best split found.  bits: caller-owned HOST buffer of split_words() words. */
typedef struct {
    uint64_t* bits;
    double fitness;
    uint32_t k;                 /* number of blocks m                          */
    int64_t var_num;            /* V = k*S2 - S1^2 = k^2 sigma^2               */
    uint64_t s1, s2;            /* sum t_j, sum t_j^2 (ns, ns^2)               */
    uint64_t overhead_ns;       /* sum of the cut overheads                    */
    double expected_wait_ns;    /* Eq. 1: S2 / (2 S1)   (P@17226-17827)        */
    uint32_t generation_found;  /* generation the record was first reached     */
    uint32_t generations_run;   /* transitions performed (< generations on stall) */
    uint64_t evaluations;       /* fitness evaluations by this handle          */
} split_best_t;

/* a1, a3-a9 — run the GA: init generation 0 from seed (re-initialises on every
 * call), then up to `generations` transitions (R11).  With islands across
 * ranks every rank must call it with the same arguments; best_out then holds
 * the GLOBAL best on every rank.  Synchronous. */
int split_ga_run(split_ga_t* h, uint32_t generations, uint64_t seed, split_best_t* best_out);

/* Copy the current population of local island `local_island` (after the last
 * split_ga_run) to host buffers bits_host[N*W] and fitness_host[N] (either may
 * be NULL).  For tests and checkpointing.  Synchronous. */
int split_ga_population(split_ga_t* h, uint32_t local_island, uint64_t* bits_host, double* fitness_host);

/* a10 — Algorithm 1 greedy preemption (host only, O(n)).  queue[0] is the head
 * (runs next), queue[n-1] the tail.  *insert_pos receives the index at which
 * the incoming request is inserted (0 = head, n = behind the tail).
 * SPLIT_E_INVAL when ext_ns <= 0, ext_left_ns not in [0, ext_ns] (any request),
 * alpha <= 0, queue == NULL with n > 0, or insert_pos == NULL.
 * Under reading R12 the decision reduces to: scanning from the tail, pass t_i
 * iff its type differs and ext_left(t_i)*ext(t_i) > ext_left(new)*ext(new). */
typedef struct {
    uint32_t type_id;
    int64_t arrival_ns, ext_ns, ext_left_ns;
} split_request;
typedef struct {
    int64_t now_ns;
    double alpha;               /* latency target = alpha * Ext (fn. 3, P@29746-29870) */
    uint32_t n;
    const split_request* queue; /* host, n entries, [0] = head */
    split_request incoming;
} split_queue_state;
int split_preempt_decide(const split_queue_state* q, uint32_t* insert_pos);

/* Block execution times of one split under the additive model of Eq. 2's
 * fitness (R2, R3): block j runs operators c_{j-1}+1 .. c_j
 * ("selects m-1 cut points to divide vanilla models into m blocks",
 * P@20780-20831), its time is the sum of their profiled latencies
 * (P@18308-18385) plus the overhead of the cut that starts it (the block after
 * cut p pays cut_overhead_ns[p]; block 1 pays nothing).  Host only, no GPU:
 * the f2 simulator's per-model block lists come from here.
 *   latencies_ns     host, n_ops >= 2 entries, each >= 0
 *   cut_overhead_ns  host, n_ops-1 entries >= 0, or NULL (all 0)
 *   bits             host, ceil((n_ops-1)/64) words, the split's cut bitset
 *                    (padding bits >= n_ops-1 ignored)
 *   out_ns           host, `cap` entries: t_1 .. t_k
 * *k receives the number of blocks (popcount + 1) even when it exceeds cap
 * (then SPLIT_E_RANGE and out_ns holds the first cap blocks).
 * SPLIT_E_INVAL: NULL pointer (out_ns may be NULL only when cap == 0),
 * n_ops < 2 or a negative latency / overhead. */
int split_block_times(const int64_t* latencies_ns, const int64_t* cut_overhead_ns, uint32_t n_ops,
                      const uint64_t* bits, int64_t* out_ns, uint32_t cap, uint32_t* k);

/* f2 — QoS simulator (R20).  Batched Monte-Carlo
 * of one edge executor serving requests of n_types split models: requests are
 * preempted only between blocks (§3.4, P@24400-26700), the queue order is
 * decided at each arrival by Algorithm 1 (policy 1, the closed form of
 * split_preempt_decide) or FIFO (policy 0), the latency target is alpha*Ext
 * (fn. 3, P@29746-29870) and a request violates it when t_ete/Ext > alpha
 * (Eq. 3, §5.2).  One replica per GPU thread; everything is integer ns.
 *   blocks_ns    host, sum(n_blocks) entries: model m's blocks in order, each in
 *                [1, 2^32); Ext(m) = sum of its blocks < 2^32
 *   n_blocks     host, n_types entries (1..65535); n_types in [1, 65535]
 *   arrival_ns   device int64 [n_req][n_rep] (request-major: request i of replica
 *                r at i*n_rep + r, so a warp's accesses coalesce), non-decreasing
 *                over i per replica, >= 0
 *   type_id      device uint32 [n_req][n_rep], < n_types
 *   alpha_milli  host, n_alpha (<= 32) thresholds alpha*1000 (> 0)
 *   t_ete_out    device int64 [n_req][n_rep]: end-to-end latency per request
 *   viol_out     device uint32 [n_rep][n_alpha]: #{i : 1000 t_ete > alpha_milli Ext}
 *   rr_out       device double [n_rep][2]: sum of t_ete/Ext and of its square,
 *                added in request order
 * Synchronous.  SPLIT_E_INVAL on bad host arguments; SPLIT_E_RANGE when a
 * replica has unordered arrivals / a bad type id, or more than 160 pending
 * requests (a batch where some replica exceeds 32 is re-run with a 160-entry
 * queue, more slowly; every output is rewritten). */
int split_qos_simulate(const int64_t* blocks_ns, const uint32_t* n_blocks, uint32_t n_types, uint32_t policy,
                       const uint32_t* alpha_milli, uint32_t n_alpha, uint64_t n_rep, uint32_t n_req,
                       const int64_t* arrival_ns, const uint32_t* type_id, int64_t* t_ete_out,
                       uint32_t* viol_out, double* rr_out, int device, void* stream);

/* f4 — elastic model splitting (§3.3 P@22612-23675:
 * "under conditions of particularly high request density, model splitting is
 * temporarily disabled ... when an excessive number of requests of the same
 * type are present, splitting is also temporarily suspended").  The paper
 * gives no thresholds, so they are arguments (reading R23): a
 * request of type m arriving when the pending queue holds >= d_max requests,
 * or >= s_max requests of type m, runs UNSPLIT — one block of unsplit_ns[m]
 * (the model without cut overheads, T) — and joins the queue tail (no
 * preemption); otherwise it is split and placed by Algorithm 1 exactly as
 * split_qos_simulate policy 1.  Queued unsplit requests take part in later
 * Algorithm 1 scans with Ext_left = unsplit_ns[m].  Violations and response
 * ratios are taken against ref_ns[m]: NULL = the same per-type Ext (sum of the
 * split blocks) as split_qos_simulate, so the two are directly comparable; or
 * e.g. ref_ns = unsplit_ns for §5.2's isolated execution time of the model
 * (then a request served unsplit has RR >= 1 and the target is alpha * T).
 * d_max = s_max = UINT32_MAX reproduces policy 1, d_max = 0 a FIFO queue of
 * unsplit models.
 *   unsplit_ns  host, n_types entries in [1, 2^32)
 *   ref_ns      host, n_types entries in [1, 2^32), or NULL
 * Other arguments, layouts, synchronisation and errors: split_qos_simulate. */
int split_qos_simulate_elastic(const int64_t* blocks_ns, const uint32_t* n_blocks, const int64_t* unsplit_ns,
                               const int64_t* ref_ns, uint32_t n_types, uint32_t d_max, uint32_t s_max,
                               const uint32_t* alpha_milli,
                               uint32_t n_alpha, uint64_t n_rep, uint32_t n_req, const int64_t* arrival_ns,
                               const uint32_t* type_id, int64_t* t_ete_out, uint32_t* viol_out, double* rr_out,
                               int device, void* stream);

/* Island communicator over NCCL (the libnccl.so.2 already loaded in the
 * process, e.g. by torch).  Rank r of `world` runs islands_per_device islands
 * starting at island_id = r*islands_per_device.  unique_id: 128 bytes from
 * rank 0, broadcast by the caller (e.g. torch.distributed).  Collective. */
int split_comm_unique_id(uint8_t out[128]);
int split_comm_init(const uint8_t id[128], int rank, int world, int device, void** comm);
void split_comm_destroy(void* comm);

/* f1 — exact optimum by exhaustive enumeration of all 2^(n_ops-1) splits
 * (the quantity the GA approximates, P@9901-10019 counts
 * 287,980 profiled candidates for 3 cuts of ResNet50).  Requires
 * n_ops - 1 <= 44 and k_max <= 64 (SPLIT_E_INVAL otherwise); the time grows as
 * 2^(n_ops-1) (about 2^40 splits per second on one B200).  best_out receives
 * the canonical best (fitness desc, bitset asc; R10) over k in [k_min, k_max]
 * with its statistics (evaluations = 2^(n_ops-1), generation fields 0);
 * best_out->bits: host buffer of split_words() words.  If min_v_per_k (host,
 * k_max+1 entries) is non-NULL it receives the minimum V = k*S2 - S1^2 over all
 * splits with k blocks (-1 where none), for k in [0, k_max]; argmin_per_k
 * (host, k_max+1) the smallest bitset attaining it.  Synchronous, on the
 * handle's stream; device scratch is allocated and freed inside the call. */
int split_exhaustive(split_ga_t* h, split_best_t* best_out, int64_t* min_v_per_k, uint64_t* argmin_per_k);

/* a0 again on a live handle: replace its chain (same n_ops) -- new per-operator
 * latencies (profiled per operator, P@18308-18385) and cut overheads (the data
 * transmission a cut adds, P@13239-13520; host, copied; NULL = 0), validated and
 * guarded exactly as split_ga_create does for the handle's k_max -- and upload
 * the tables stream-ordered on the handle's stream.  No allocation: the serving
 * path re-splits a model whose profile changed without create/destroy.  The
 * population is invalidated (split_ga_run re-initialises anyway).
 * SPLIT_E_INVAL / SPLIT_E_RANGE as in split_ga_create. */
int split_ga_set_chain(split_ga_t* h, const int64_t* latencies_ns, const int64_t* cut_overhead_ns);

/* f3 — Eq. 1-driven choice of the block count (R21).
 * Runs the fixed-k GA (k_min = k_max = k, `generations`, `seed`) for every k
 * in [k_lo, k_hi] (1 <= k_lo <= k_hi <= the handle's k_max) and reports each
 * run's best split: Eq. 2 fitness, Eq. 1's expected wait S2/(2 S1) of a short
 * request arriving during the model (P@17226-17827), overheads, V, S1, S2 and
 * the block-count criterion cost_ns = S2/(2 S1) + OV: the short request's wait
 * plus the latency the cuts add to the split request itself ("an optimal
 * number of splits exists and more blocks may not be beneficial",
 * P@18542-18830).  *k_best = the k of minimum cost (compared exactly in
 * integers; ties -> the smaller k; 0 if no k has a feasible split; cost_ns =
 * +INF for an infeasible k).  out: host, k_hi-k_lo+1 entries.
 * Synchronous; the handle's own k range is restored afterwards. */
typedef struct {
    uint32_t k;
    double fitness;
    double expected_wait_ns;
    uint64_t overhead_ns;
    int64_t var_num;
    uint64_t s1, s2;
    double cost_ns;
} split_k_result;
int split_k_sweep(split_ga_t* h, uint32_t k_lo, uint32_t k_hi, uint32_t generations, uint64_t seed,
                  split_k_result* out, uint32_t* k_best);

/* f1 — minimum S2 = sum t_j^2 over all k-block splits, k = 1..k_max, by the
 * O(k n^2) dynamic program D[j][i] = min_p D[j-1][p] + (P[i]-P[p]+ovh[p-1])^2
 * (one CTA on the handle's device).  Exact for any per-cut overheads; with a
 * constant overhead delta, S1 = T + (k-1) delta is fixed and
 * V*_k = k*S2*_k - S1^2 is the minimum variance.  s2_out: host,
 * k_max+1 entries ([0] = UINT64_MAX; UINT64_MAX where k > n_ops).
 * 1 <= k_max <= the handle's k_max (the create-time guard keeps every sum in
 * range).  Synchronous. */
int split_dp_min_s2(split_ga_t* h, uint32_t k_max, uint64_t* s2_out);

/* f1 — the two-cut map, synthetic analog of Fig. 2 (P@11560-12128: "the
 * relationship of splitting overhead and standard deviation to position of cut
 * points.  The X-axis and Y-axis show position of the first cut point and the
 * second cut point"; §3.1 P@15908-16933).  For every pair of cut positions
 * a <= b in [0, n_ops-2] the split with cuts {a, b} (3 blocks; a == b: the
 * one-cut split {a}, 2 blocks) under the handle's chain: V = k S2 - S1^2
 * (= k^2 sigma^2, exact), OV = the cut overheads (splitting overhead =
 * OV / T, fn. 2) and the Eq. 2 fitness (no block-count restriction).
 * Outputs: DEVICE buffers of (n_ops-1)^2 entries, row-major, entry [a][b] at
 * a*(n_ops-1)+b, 8-byte aligned; a > b gets V = -1, OV = 0, fitness =
 * -INFINITY; any output may be NULL.  Asynchronous on the handle's stream;
 * caller-owned buffers.  SPLIT_E_INVAL when the handle's k_max < 3 (its
 * create-time guards must cover two cuts). */
int split_heatmap2(split_ga_t* h, int64_t* var_out, uint64_t* ov_out, double* fit_out);

void split_ga_destroy(split_ga_t* h);
const char* split_strerror(int code);
const char* split_last_error(void);

/* Diagnostics (device self-tests used by the parity tests): evaluate the
 * device Philox4x32-10 on n (ctr[4], key[2]) tuples and the device dexp on n
 * doubles.  Host buffers; synchronous.  device = CUDA ordinal. */
int split_selftest_philox(int device, const uint32_t* ctr_key /* n*6 */, uint32_t n, uint32_t* out /* n*4 */);
int split_selftest_dexp(int device, const double* z, uint32_t n, double* out);

/* Timing support for bench.py: number of kernel launches the last
 * split_ga_run / split_eval_batch issued, and the device time (ms, CUDA events
 * on the handle's stream) of the last split_ga_run's generation loop and of its
 * dominant kernel. */
typedef struct {
    uint64_t launches;
    float ms_total;
    float ms_loop;
    uint32_t general_selects;   /* generations that needed the radix top-E path */
    uint32_t fast_selects;      /* generations served by the candidate merge     */
} split_run_stats;
int split_last_run_stats(const split_ga_t* h, split_run_stats* out);

#ifdef __cplusplus
}
#endif
#endif /* SPLIT_GA_H */
