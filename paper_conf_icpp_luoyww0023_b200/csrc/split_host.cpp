// split_host.cpp — C ABI of include/split_ga.h: validation, chain staging (a0),
// the GA driver around the persistent kernel (segments, sync points, island
// migration over NCCL), best-record assembly, Algorithm 1 (a10, host only).
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <math.h>
#include <nccl.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <new>
#include <vector>

#include "split_ga.h"
#include "split_internal.h"

using namespace splitga;

// ------------------------------------------------------------------------
// errors
// ------------------------------------------------------------------------
static thread_local char g_err[512];

static int fail(int code, const char* fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return code;
}

#define CU(call)                                                                                  \
    do {                                                                                          \
        cudaError_t e_ = (call);                                                                  \
        if (e_ != cudaSuccess)                                                                    \
            return fail(SPLIT_E_CUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
    } while (0)

extern "C" const char* split_last_error(void) { return g_err; }

extern "C" const char* split_strerror(int code)
{
    switch (code) {
    case SPLIT_OK: return "ok";
    case SPLIT_E_INVAL: return "invalid argument";
    case SPLIT_E_RANGE: return "latency/overhead magnitudes exceed the exact-integer guards";
    case SPLIT_E_ALIGN: return "misaligned device buffer";
    case SPLIT_E_NOMEM: return "out of memory";
    case SPLIT_E_CUDA: return "CUDA error";
    case SPLIT_E_NCCL: return "NCCL error";
    case SPLIT_E_STATE: return "invalid state";
    default: return "unknown error";
    }
}

// ------------------------------------------------------------------------
// NCCL, resolved at run time from the libnccl.so.2 already in the process
// (torch's), so the library never pins a second NCCL build.
// ------------------------------------------------------------------------
struct NcclApi {
    ncclResult_t (*getUniqueId)(ncclUniqueId*);
    ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int);
    ncclResult_t (*allGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t);
    ncclResult_t (*commDestroy)(ncclComm_t);
    const char* (*getErrorString)(ncclResult_t);
    bool ok;
};

static NcclApi* nccl_api()
{
    static NcclApi api{};
    static bool tried = false;
    if (tried) return api.ok ? &api : nullptr;
    tried = true;
    void* h = nullptr;
    const char* env = getenv("SPLIT_NCCL_LIB");
    if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_LOCAL);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_LOCAL);
    if (!h) return nullptr;
    api.getUniqueId = (decltype(api.getUniqueId))dlsym(h, "ncclGetUniqueId");
    api.commInitRank = (decltype(api.commInitRank))dlsym(h, "ncclCommInitRank");
    api.allGather = (decltype(api.allGather))dlsym(h, "ncclAllGather");
    api.commDestroy = (decltype(api.commDestroy))dlsym(h, "ncclCommDestroy");
    api.getErrorString = (decltype(api.getErrorString))dlsym(h, "ncclGetErrorString");
    api.ok = api.getUniqueId && api.commInitRank && api.allGather && api.commDestroy && api.getErrorString;
    return api.ok ? &api : nullptr;
}

struct SplitComm {
    ncclComm_t comm;
    int rank, world, device;
};

extern "C" int split_comm_unique_id(uint8_t out[128])
{
    if (!out) return fail(SPLIT_E_INVAL, "split_comm_unique_id: out is NULL");
    NcclApi* api = nccl_api();
    if (!api) return fail(SPLIT_E_NCCL, "libnccl.so.2 not loadable (set SPLIT_NCCL_LIB)");
    ncclUniqueId id;
    ncclResult_t r = api->getUniqueId(&id);
    if (r != ncclSuccess) return fail(SPLIT_E_NCCL, "ncclGetUniqueId: %s", api->getErrorString(r));
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    memcpy(out, &id, 128);
    return SPLIT_OK;
}

extern "C" int split_comm_init(const uint8_t id[128], int rank, int world, int device, void** comm)
{
    if (!id || !comm || world < 1 || rank < 0 || rank >= world) return fail(SPLIT_E_INVAL, "split_comm_init: bad args");
    NcclApi* api = nccl_api();
    if (!api) return fail(SPLIT_E_NCCL, "libnccl.so.2 not loadable (set SPLIT_NCCL_LIB)");
    CU(cudaSetDevice(device));
    ncclUniqueId uid;
    memcpy(&uid, id, 128);
    SplitComm* c = new (std::nothrow) SplitComm{};
    if (!c) return fail(SPLIT_E_NOMEM, "split_comm_init: host alloc");
    ncclResult_t r = api->commInitRank(&c->comm, world, uid, rank);
    if (r != ncclSuccess) {
        delete c;
        return fail(SPLIT_E_NCCL, "ncclCommInitRank: %s", api->getErrorString(r));
    }
    c->rank = rank;
    c->world = world;
    c->device = device;
    *comm = c;
    return SPLIT_OK;
}

extern "C" void split_comm_destroy(void* comm)
{
    if (!comm) return;
    SplitComm* c = (SplitComm*)comm;
    NcclApi* api = nccl_api();
    if (api) api->commDestroy(c->comm);
    delete c;
}

// ------------------------------------------------------------------------
// handle
// ------------------------------------------------------------------------
struct split_ga_t {
    split_ga_params p;
    uint32_t n, W;
    uint64_t T;
    int device;
    cudaStream_t stream;
    int num_sms;
    ChainDev ch;
    GaArgs ga;
    int grid;
    uint32_t cpi;
    std::vector<void*> allocs;
    // host-side state
    uint32_t last_gen;
    bool have_pop;
    split_run_stats stats;
    // scratch
    int64_t* d_stats;
    double* d_statf;
    uint64_t* d_bits1;
    cudaEvent_t ev[4];
    unsigned long long* d_trace;   // SPLIT_TRACE=<csv path>: phase timestamps of the first RUN segment
    uint32_t trace_gens;
    // host copy of the chain words: P[0..n] | ovh[0..n-2] (f1 exact solvers)
    std::vector<uint32_t> hwords;
    uint32_t p_words;
    // eval_batch_host staging
    uint64_t* d_hbits[2];
    double* d_hfit[2];
    uint64_t h_chunk;
    cudaStream_t hs[2];
};

extern "C" void split_ga_params_default(split_ga_params* p)
{
    if (!p) return;
    memset(p, 0, sizeof(*p));
    p->pop_size = 65536;
    p->n_elite = 1024;
    p->tournament_size = 4;
    p->p_crossover = 0.9;
    p->p_mutation = 0.2;
    p->k_min = 2;
    p->k_max = 32;
    p->front_skip = 0;
    p->stall_generations = 0;
    p->cut_overhead_ns = nullptr;
    p->island_id = 0;
    p->n_islands = 1;
    p->islands_per_device = 1;
    p->migration_interval = 0;
    p->n_migrants = 0;
    p->comm = nullptr;
    p->device = 0;
    p->stream = nullptr;
}

extern "C" uint32_t split_words(const split_ga_t* h) { return h ? h->W : 0; }

static void free_all(split_ga_t* h)
{
    for (void* q : h->allocs) cudaFree(q);
    h->allocs.clear();
    for (int i = 0; i < 4; ++i)
        if (h->ev[i]) cudaEventDestroy(h->ev[i]);
    for (int i = 0; i < 2; ++i)
        if (h->hs[i]) cudaStreamDestroy(h->hs[i]);
}

template <class T>
static int dalloc(split_ga_t* h, T** out, size_t count)
{
    void* q = nullptr;
    size_t bytes = count * sizeof(T);
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMalloc(&q, bytes);
    if (e != cudaSuccess) return fail(SPLIT_E_NOMEM, "cudaMalloc(%zu): %s", bytes, cudaGetErrorString(e));
    h->allocs.push_back(q);
    e = cudaMemset(q, 0, bytes);
    if (e != cudaSuccess) return fail(SPLIT_E_CUDA, "cudaMemset: %s", cudaGetErrorString(e));
    *out = (T*)q;
    return SPLIT_OK;
}

// Device arena: create() plans every buffer, then makes ONE cudaMalloc and one
// stream-ordered memset (dozens of separate cudaMalloc/cudaMemset calls cost
// milliseconds per handle, which the end-to-end path pays on every create).
struct DevPlan {
    std::vector<std::pair<void**, size_t>> req;
    template <class T>
    void add(T** out, size_t count)
    {
        *out = nullptr;
        req.push_back({(void**)out, std::max<size_t>(count * sizeof(T), 16)});
    }
};

static int commit_plan(split_ga_t* h, DevPlan& pl)
{
    size_t total = 0;
    for (auto& r : pl.req) total = ((total + 255) & ~(size_t)255) + r.second;
    void* base = nullptr;
    cudaError_t e = cudaMalloc(&base, total);
    if (e != cudaSuccess) return fail(SPLIT_E_NOMEM, "cudaMalloc(%zu): %s", total, cudaGetErrorString(e));
    h->allocs.push_back(base);
    size_t off = 0;
    for (auto& r : pl.req) {
        off = (off + 255) & ~(size_t)255;
        *r.first = (uint8_t*)base + off;
        off += r.second;
    }
    e = cudaMemsetAsync(base, 0, total, h->stream);
    if (e != cudaSuccess) return fail(SPLIT_E_CUDA, "cudaMemsetAsync: %s", cudaGetErrorString(e));
    pl.req.clear();
    return SPLIT_OK;
}

static uint64_t bern_thr(double p)
{
    if (!(p > 0.0)) return 0;
    if (p >= 1.0) return (uint64_t)1 << 32;
    return (uint64_t)floor(p * 4294967296.0);
}

static uint32_t pow2_at_least(uint32_t x)
{
    uint32_t p = 1;
    while (p < x) p <<= 1;
    return p;
}

#define TRY(x)                  \
    do {                        \
        int rc_ = (x);          \
        if (rc_ != SPLIT_OK) {  \
            free_all(h);        \
            delete h;           \
            return rc_;         \
        }                       \
    } while (0)

// a0: host tables of one chain -- P and ovh words, the {P[p+1], ovh[p]} pairs, the
// Eq. 2 reciprocals -- after validation and the exact-integer guards for k_max.
struct ChainHost {
    std::vector<uint32_t> words, po;
    std::vector<double> rcp;
    uint32_t p_words = 0, o_words = 0;
    uint64_t T = 0;
};

static int chain_tables(const int64_t* lat, const int64_t* ovh_in, uint32_t n, uint32_t k_max, ChainHost& c)
{
    unsigned __int128 T = 0;
    for (uint32_t i = 0; i < n; ++i) {
        if (lat[i] < 0) return fail(SPLIT_E_INVAL, "latencies_ns[%u] < 0", i);
        T += (uint64_t)lat[i];
    }
    if (T < 1) return fail(SPLIT_E_INVAL, "sum of latencies must be >= 1");
    std::vector<int64_t> ovh(n - 1, 0);
    if (ovh_in) {
        for (uint32_t i = 0; i + 1 < n; ++i) {
            if (ovh_in[i] < 0) return fail(SPLIT_E_INVAL, "cut_overhead_ns[%u] < 0", i);
            ovh[i] = ovh_in[i];
        }
    }
    // exact-integer guards (a0)
    std::vector<int64_t> srt(ovh);
    std::sort(srt.begin(), srt.end(), std::greater<int64_t>());
    unsigned __int128 Tp = T;
    for (uint32_t i = 0; i + 1 < k_max && i < srt.size(); ++i) Tp += (uint64_t)srt[i];
    if (Tp >= ((unsigned __int128)1 << 32)) return fail(SPLIT_E_RANGE, "T + largest overheads must be < 2^32 ns");
    if ((unsigned __int128)(k_max - 1) * Tp * Tp >= ((unsigned __int128)1 << 63))
        return fail(SPLIT_E_RANGE, "(k_max-1) * T'^2 must be < 2^63");
    // chain words: P[0..n] padded to x4, ovh[0..n-2] padded to x4
    c.p_words = (n + 1 + 3) & ~3u;
    c.o_words = (n - 1 + 3) & ~3u;
    c.words.assign(c.p_words + c.o_words, 0);
    uint64_t acc = 0;
    for (uint32_t i = 0; i < n; ++i) {
        c.words[i] = (uint32_t)acc;
        acc += (uint64_t)lat[i];
    }
    c.words[n] = (uint32_t)acc;
    for (uint32_t i = 0; i + 1 < n; ++i) c.words[c.p_words + i] = (uint32_t)ovh[i];
    // interleaved {P[p+1], ovh[p]} table for the eval kernel's walk
    const uint32_t po_n = ((n - 1) + 1) & ~1u;                  // entries, even -> 16-byte multiple
    c.po.assign(2 * (size_t)po_n, 0);
    for (uint32_t q = 0; q + 1 < n; ++q) {
        c.po[2 * q] = c.words[q + 1];
        c.po[2 * q + 1] = (uint32_t)ovh[q];
    }
    // Eq. 2 reciprocals (ChainDev::rcp): IEEE divisions, i.e. correctly rounded
    c.rcp.assign(2 * (size_t)n + 2, 0.0);
    c.rcp[0] = 1.0 / (double)acc;
    for (uint32_t k = 1; k <= n; ++k) {
        c.rcp[k] = 1.0 / (double)k;
        c.rcp[n + 1 + k] = 1.0 / ((double)k * (double)acc);   // k T < 2^53: exact product
    }
    c.T = acc;
    return SPLIT_OK;
}

extern "C" int split_ga_create(const int64_t* lat, uint32_t n, const split_ga_params* pp, split_ga_t** out)
{
    if (!lat || !pp || !out) return fail(SPLIT_E_INVAL, "split_ga_create: NULL argument");
    const split_ga_params p = *pp;
    if (n < 2 || n > 64u * kMaxWords + 1) return fail(SPLIT_E_INVAL, "n_ops must be in [2, %u]", 64u * kMaxWords + 1);
    if (p.pop_size < 2) return fail(SPLIT_E_INVAL, "pop_size must be >= 2");
    if (p.n_elite > p.pop_size || p.n_elite > kMaxElite) return fail(SPLIT_E_INVAL, "n_elite must be <= min(N, %u)", kMaxElite);
    if ((p.pop_size - p.n_elite) & 1u) return fail(SPLIT_E_INVAL, "pop_size - n_elite must be even");
    if (p.tournament_size < 1 || p.tournament_size > 32) return fail(SPLIT_E_INVAL, "tournament_size must be in [1, 32]");
    if (!(p.p_crossover >= 0.0 && p.p_crossover <= 1.0) || !(p.p_mutation >= 0.0 && p.p_mutation <= 1.0))
        return fail(SPLIT_E_INVAL, "probabilities must be in [0, 1]");
    if (p.k_min < 1 || p.k_min > p.k_max || p.k_max > n) return fail(SPLIT_E_INVAL, "need 1 <= k_min <= k_max <= n_ops");
    if (p.front_skip > n - 2 || p.k_max - 1 > n - 1 - p.front_skip)
        return fail(SPLIT_E_INVAL, "k_max - 1 cut points do not fit in [front_skip, n_ops-2]");
    if (p.islands_per_device < 1 || p.islands_per_device > kMaxLocalIslands)
        return fail(SPLIT_E_INVAL, "islands_per_device must be in [1, %u]", kMaxLocalIslands);
    if (p.n_islands < p.islands_per_device || p.island_id + p.islands_per_device > p.n_islands)
        return fail(SPLIT_E_INVAL, "island range outside [0, n_islands)");
    if ((uint64_t)p.n_islands * p.pop_size >= (1ull << 32)) return fail(SPLIT_E_INVAL, "n_islands * pop_size must be < 2^32");
    if (p.n_islands > p.islands_per_device && !p.comm)
        return fail(SPLIT_E_INVAL, "islands span ranks but comm is NULL");
    if (p.comm) {
        // the all-gathers write world * islands_per_device slots at rank * islands_per_device:
        // any other layout would make NCCL write past (or into the wrong slots of) the buffers
        const SplitComm* c = (const SplitComm*)p.comm;
        if (p.n_islands != (uint32_t)c->world * p.islands_per_device || p.island_id != (uint32_t)c->rank * p.islands_per_device)
            return fail(SPLIT_E_INVAL, "comm of rank %d / world %d needs n_islands = world*islands_per_device and "
                        "island_id = rank*islands_per_device (got %u, %u)", c->rank, c->world, p.n_islands, p.island_id);
        if (c->device != p.device)
            return fail(SPLIT_E_INVAL, "comm is bound to device %d, params.device is %d", c->device, p.device);
    }
    const bool migrate = p.migration_interval > 0 && p.n_islands > 1;
    if (migrate && (p.n_migrants < 1 || p.n_migrants > p.pop_size - p.n_elite || p.n_migrants > kMaxElite))
        return fail(SPLIT_E_INVAL, "n_migrants must be in [1, min(N - E, %u)]", kMaxElite);
    ChainHost chn;
    {
        const int rc = chain_tables(lat, p.cut_overhead_ns, n, p.k_max, chn);
        if (rc != SPLIT_OK) return rc;
    }
    const uint64_t T = chn.T;

    split_ga_t* h = new (std::nothrow) split_ga_t();
    if (!h) return fail(SPLIT_E_NOMEM, "host alloc");
    h->p = p;
    h->p.cut_overhead_ns = nullptr;
    h->n = n;
    h->W = (n - 1 + 63) / 64;
    h->T = (uint64_t)T;
    h->device = p.device;
    h->stream = (cudaStream_t)p.stream;
    {
        cudaError_t e = cudaSetDevice(p.device);
        if (e == cudaSuccess) e = cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, p.device);
        if (e != cudaSuccess) {
            delete h;
            return fail(SPLIT_E_CUDA, "device %d: %s", p.device, cudaGetErrorString(e));
        }
    }
    std::vector<uint32_t>& words = chn.words;
    std::vector<uint32_t>& po = chn.po;
    std::vector<double>& rcp = chn.rcp;
    const uint32_t p_words = chn.p_words, o_words = chn.o_words;
    const uint64_t acc = chn.T;
    DevPlan plan;
    uint32_t* d_chain = nullptr;
    uint32_t* d_po = nullptr;
    double* d_rcp = nullptr;
    plan.add(&d_chain, words.size());
    plan.add(&d_po, po.size());
    plan.add(&d_rcp, rcp.size());
    h->hwords = words;
    h->p_words = p_words;
    ChainDev& ch = h->ch;
    ch.po_bytes = (uint32_t)(po.size() * 4);
    ch.n = n;
    ch.W = h->W;
    ch.p_words = p_words;
    ch.o_words = o_words;
    ch.T = (uint32_t)acc;
    ch.k_min = p.k_min;
    ch.k_max = p.k_max;
    const uint32_t rem = (n - 1) & 63u;
    ch.last_mask = rem ? ((1ull << rem) - 1) : ~0ull;

    GaArgs& a = h->ga;
    memset(&a, 0, sizeof(a));
    a.ch = ch;
    a.N = p.pop_size;
    a.E = p.n_elite;
    a.s = p.tournament_size;
    a.K = migrate ? p.n_migrants : 0;
    a.I = p.islands_per_device;
    a.island_base = p.island_id;
    a.I_total = p.n_islands;
    a.front_skip = p.front_skip;
    a.stall = p.stall_generations;
    a.thr_c = bern_thr(p.p_crossover);
    a.thr_m = bern_thr(p.p_mutation);
    uint32_t sc = std::max<uint32_t>(pow2_at_least(std::max(kCandCap, std::max(kWorstCap, kWorstSample))),
                                     pow2_at_least(std::max<uint32_t>(a.E, 2)));
    if (migrate) sc = std::max(sc, pow2_at_least((p.n_islands - 1) * a.K));
    a.sort_cap = sc;
    a.Ns = (a.N + 3u) & ~3u;
    // size the per-CTA partial arrays for the largest grid the launch bounds allow,
    // then take the real co-resident grid from the occupancy calculator
    {
        const uint32_t grid_max = (uint32_t)(ga_max_blocks_per_sm(h->W) * h->num_sms);
        if (grid_max < 2 * a.I) {
            const int sms = h->num_sms;          // read before h is freed
            free_all(h);
            delete h;
            return fail(SPLIT_E_INVAL, "too many islands per device for %d SMs", sms);
        }
        a.cpi = (grid_max - a.I) / a.I;
        a.cpi_pad = (a.cpi + 3u) & ~3u;
        a.stage_bits = (size_t)a.cpi_pad * h->W * 8 <= 16384 ? 1u : 0u;
    }
    if (const size_t smem = ga_smem_bytes(a); smem > 227 * 1024) {
        free_all(h);
        delete h;
        return fail(SPLIT_E_INVAL, "shared-memory plan %zu B exceeds 227 KB (n_ops, islands or migrants too large)",
                    smem);
    }
    cudaError_t ge;
    h->grid = ga_grid(a, h->num_sms, &ge);
    if (ge != cudaSuccess || h->grid < 2 * (int)a.I) {
        const int grid = h->grid;               // read before h is freed
        free_all(h);
        delete h;
        return fail(SPLIT_E_CUDA, "GA kernel occupancy: %s (grid %d)", cudaGetErrorString(ge), grid);
    }
    a.cpi = (uint32_t)(h->grid - (int)a.I) / a.I;     // <= the sizing value; cpi_pad keeps its value
    h->cpi = a.cpi;
    const size_t IN = (size_t)a.I * a.N, INs = (size_t)a.I * a.Ns;
    for (int b = 0; b < 2; ++b) {
        plan.add(&a.pop[b], IN * h->W);
        plan.add(&a.fit[b], INs);
    }
    {
        // candidate regions: worker CTA c of an island produces at most 32 children per
        // chunk it is dealt (chunks round-robin over cpi CTAs x warps)
        const uint32_t chunks = (a.N - a.E + 31u) / 32u;
        a.creg = 32u * ((chunks + a.cpi - 1u) / a.cpi) + 32u;
    }
    for (int b = 0; b < 3; ++b) {
        plan.add(&a.cand_key[b], (size_t)a.I * a.cpi * a.creg);
        plan.add(&a.cand_idx[b], (size_t)a.I * a.cpi * a.creg);
    }
    plan.add(&a.cand_cnt, 3 * (size_t)a.I * a.cpi_pad);
    plan.add(&a.rc_cnt, ((3 * (size_t)a.I + 3) & ~(size_t)3) + 4);
    for (int b = 0; b < 3; ++b) plan.add(&a.rc_idx[b], INs);
    plan.add(&a.snap_f, 2 * (size_t)a.I);
    plan.add(&a.snap_bits, 2 * (size_t)a.I * h->W);
    plan.add(&a.sel_key, (size_t)a.I * kMaxElite);
    plan.add(&a.sel_idx, (size_t)a.I * kMaxElite);
    plan.add(&a.sel_cnt, a.I);
    plan.add(&a.tau, 2 * (size_t)a.I);
    plan.add(&a.ghist, 3 * (size_t)a.I * 256);
    plan.add(&a.part_f, 2 * (size_t)a.I * a.cpi_pad);
    plan.add(&a.part_idx, 2 * (size_t)a.I * a.cpi_pad);
    plan.add(&a.part_bits, 2 * (size_t)a.I * a.cpi_pad * h->W);
    plan.add(&a.rec_f, a.I);
    plan.add(&a.rec_bits, (size_t)a.I * h->W);
    plan.add(&a.rec_gen, a.I);
    plan.add(&a.rec_valid, a.I);
    a.xstride = a.K * h->W + a.K + 2 + h->W;
    plan.add(&a.xch, (size_t)a.I_total * a.xstride);
    plan.add(&a.rk_key, (size_t)a.I * kMaxElite);
    plan.add(&a.rk_idx, (size_t)a.I * kMaxElite);
    plan.add(&a.wslot, (size_t)a.I * kMaxElite);
    plan.add(&a.wthr, a.I);
    plan.add(&a.wl_key, (size_t)a.I * kWorstCap);
    plan.add(&a.wl_idx, (size_t)a.I * kWorstCap);
    plan.add(&a.wl_cnt, a.I);
    plan.add(&a.ctl, 1);
    plan.add(&a.gbar, 4);
    plan.add(&h->d_stats, 8);
    plan.add(&h->d_statf, 1);
    plan.add(&h->d_bits1, h->W);
    if (getenv("SPLIT_TRACE")) {
        h->trace_gens = 64;
        plan.add(&h->d_trace, (size_t)h->trace_gens * 16 + kTraceArrGens * 1024);   // + per-CTA arrivals
    }
    TRY(commit_plan(h, plan));
    ch.po = (const uint2*)d_po;
    ch.words = d_chain;
    ch.rcp = d_rcp;
    a.ch = ch;
    {
        cudaError_t e = cudaMemcpyAsync(d_chain, words.data(), words.size() * 4, cudaMemcpyHostToDevice, h->stream);
        if (e == cudaSuccess) e = cudaMemcpyAsync(d_po, po.data(), po.size() * 4, cudaMemcpyHostToDevice, h->stream);
        if (e == cudaSuccess) e = cudaMemcpyAsync(d_rcp, rcp.data(), rcp.size() * 8, cudaMemcpyHostToDevice, h->stream);
        // (pageable sources: the calls return once the host data has been staged)
        if (e != cudaSuccess) TRY(fail(SPLIT_E_CUDA, "chain upload: %s", cudaGetErrorString(e)));
    }
    for (int i = 0; i < 4; ++i) {
        cudaError_t e = cudaEventCreate(&h->ev[i]);
        if (e != cudaSuccess) TRY(fail(SPLIT_E_CUDA, "cudaEventCreate: %s", cudaGetErrorString(e)));
    }
    *out = h;
    return SPLIT_OK;
}

extern "C" int split_ga_set_chain(split_ga_t* h, const int64_t* lat, const int64_t* cut_overhead_ns)
{
    if (!h || !lat) return fail(SPLIT_E_INVAL, "split_ga_set_chain: NULL argument");
    ChainHost chn;
    {
        const int rc = chain_tables(lat, cut_overhead_ns, h->n, h->p.k_max, chn);
        if (rc != SPLIT_OK) return rc;
    }
    CU(cudaSetDevice(h->device));
    CU(cudaMemcpyAsync((void*)h->ch.words, chn.words.data(), chn.words.size() * 4, cudaMemcpyHostToDevice, h->stream));
    CU(cudaMemcpyAsync((void*)h->ch.po, chn.po.data(), chn.po.size() * 4, cudaMemcpyHostToDevice, h->stream));
    CU(cudaMemcpyAsync((void*)h->ch.rcp, chn.rcp.data(), chn.rcp.size() * 8, cudaMemcpyHostToDevice, h->stream));
    h->T = chn.T;
    h->ch.T = (uint32_t)chn.T;
    h->ga.ch.T = (uint32_t)chn.T;
    h->hwords = chn.words;
    h->have_pop = false;
    return SPLIT_OK;
}

// f3: Eq. 1-driven choice of the block count (reading R21).  Eq. 1
// (P@17226-17827) gives the expected wait of a short request arriving while the
// split model runs, S2 / (2 S1) = (sigma^2/t_bar + t_bar) / 2: more blocks shrink
// t_bar, but every cut adds its overhead to the split request itself ("the
// relationship between splitting overhead and average latency is hyperbolic,
// indicating that an optimal number of splits exists and more blocks may not be
// beneficial", P@18542-18830).  The criterion of a k is therefore
//     J(k) = S2/(2 S1) + OV        (short request's Eq. 1 wait + the long one's added latency)
// of the best split the fixed-k GA finds for it (same seed and budget per k);
// k* = argmin J, ties -> the smaller k, k without a feasible split skipped.  The
// comparison is exact: J = (S2 + 2 S1 OV) / (2 S1), cross-multiplied in 128 bits
// (S2 < 2^63, S1 OV < 2^64, S1 < 2^32).  With a constant per-cut overhead
// delta, S1 = T + (k-1) delta and OV = (k-1) delta are fixed per k, so J is
// minimised by the minimum-S2 split and k* equals the exact DP's whenever every
// run reaches the DP optimum.
static bool kcost_less(uint64_t s2a, uint64_t s1a, uint64_t ova, uint64_t s2b, uint64_t s1b, uint64_t ovb)
{
    const unsigned __int128 na = (unsigned __int128)s2a + 2 * (unsigned __int128)s1a * ova;
    const unsigned __int128 nb = (unsigned __int128)s2b + 2 * (unsigned __int128)s1b * ovb;
    // na / (2 s1a) < nb / (2 s1b)  <=>  na * s1b < nb * s1a  (all < 2^97)
    return na * s1b < nb * s1a;
}

extern "C" int split_k_sweep(split_ga_t* h, uint32_t k_lo, uint32_t k_hi, uint32_t generations, uint64_t seed,
                             split_k_result* out, uint32_t* k_best)
{
    if (!h || !out || !k_best) return fail(SPLIT_E_INVAL, "split_k_sweep: NULL argument");
    if (k_lo < 1 || k_lo > k_hi || k_hi > h->p.k_max)
        return fail(SPLIT_E_INVAL, "split_k_sweep: need 1 <= k_lo <= k_hi <= handle k_max = %u", h->p.k_max);
    const uint32_t kmin0 = h->ch.k_min, kmax0 = h->ch.k_max;
    std::vector<uint64_t> bits(h->W ? h->W : 1);
    int rc = SPLIT_OK;
    *k_best = 0;
    uint64_t b_s2 = 0, b_s1 = 1, b_ov = 0;
    for (uint32_t k = k_lo; k <= k_hi && rc == SPLIT_OK; ++k) {
        h->ch.k_min = h->ch.k_max = k;
        h->ga.ch.k_min = h->ga.ch.k_max = k;
        split_best_t b;
        memset(&b, 0, sizeof(b));
        b.bits = bits.data();
        rc = split_ga_run(h, generations, seed, &b);
        if (rc != SPLIT_OK) break;
        split_k_result& r = out[k - k_lo];
        r.k = k;
        r.fitness = b.fitness;
        r.expected_wait_ns = b.expected_wait_ns;
        r.overhead_ns = b.overhead_ns;
        r.var_num = b.var_num;
        r.s1 = b.s1;
        r.s2 = b.s2;
        const bool feasible = b.fitness > -INFINITY;
        r.cost_ns = feasible ? b.expected_wait_ns + (double)b.overhead_ns : INFINITY;
        if (feasible && (*k_best == 0 || kcost_less(b.s2, b.s1, b.overhead_ns, b_s2, b_s1, b_ov))) {
            *k_best = k;
            b_s2 = b.s2;
            b_s1 = b.s1;
            b_ov = b.overhead_ns;
        }
    }
    h->ch.k_min = h->ga.ch.k_min = kmin0;
    h->ch.k_max = h->ga.ch.k_max = kmax0;
    return rc;
}

extern "C" void split_ga_destroy(split_ga_t* h)
{
    if (!h) return;
    cudaSetDevice(h->device);
    cudaStreamSynchronize(h->stream);
    free_all(h);
    delete h;
}

// ------------------------------------------------------------------------
// a2 eval
// ------------------------------------------------------------------------
extern "C" int split_eval_batch(split_ga_t* h, const uint64_t* bits, uint64_t n_cand, double* out)
{
    if (!h) return fail(SPLIT_E_INVAL, "split_eval_batch: NULL handle");
    if (n_cand == 0) return SPLIT_OK;
    if (!bits || !out) return fail(SPLIT_E_INVAL, "split_eval_batch: NULL buffer");
    if (((uintptr_t)bits & 15u) || ((uintptr_t)out & 7u)) return fail(SPLIT_E_ALIGN, "bitsets must be 16-byte aligned, fitness 8-byte");
    cudaPointerAttributes at;
    memset(&at, 0, sizeof(at));             // a failed query leaves it untouched: type reads as unregistered
    if (cudaPointerGetAttributes(&at, bits) != cudaSuccess || at.type != cudaMemoryTypeDevice) {
        cudaGetLastError();
        if (!(at.type == cudaMemoryTypeManaged)) return fail(SPLIT_E_INVAL, "cut_bitsets is not a device pointer");
    }
    CU(cudaSetDevice(h->device));
    h->stats.launches = 0;
    CU(launch_eval_batch(h->ch, bits, n_cand, out, h->stream, h->num_sms, &h->stats.launches));
    return SPLIT_OK;
}

extern "C" int split_eval_batch_host(split_ga_t* h, const uint64_t* bits_host, uint64_t n_cand, double* fit_host)
{
    if (!h) return fail(SPLIT_E_INVAL, "split_eval_batch_host: NULL handle");
    if (n_cand == 0) return SPLIT_OK;
    if (!bits_host || !fit_host) return fail(SPLIT_E_INVAL, "split_eval_batch_host: NULL buffer");
    CU(cudaSetDevice(h->device));
    const uint64_t chunk = 1ull << 22;  // candidates per pipeline stage
    if (h->h_chunk == 0) {
        for (int b = 0; b < 2; ++b) {
            int rc = dalloc(h, &h->d_hbits[b], chunk * h->W);
            if (rc) return rc;
            rc = dalloc(h, &h->d_hfit[b], chunk);
            if (rc) return rc;
            CU(cudaStreamCreateWithFlags(&h->hs[b], cudaStreamNonBlocking));
        }
        h->h_chunk = chunk;
    }
    CU(cudaStreamSynchronize(h->stream));
    h->stats.launches = 0;
    for (uint64_t c = 0, k = 0; c < n_cand; c += chunk, ++k) {
        const int b = (int)(k & 1);
        const uint64_t m = std::min<uint64_t>(chunk, n_cand - c);
        CU(cudaMemcpyAsync(h->d_hbits[b], bits_host + c * h->W, m * h->W * 8, cudaMemcpyHostToDevice, h->hs[b]));
        CU(launch_eval_batch(h->ch, h->d_hbits[b], m, h->d_hfit[b], h->hs[b], h->num_sms, &h->stats.launches));
        CU(cudaMemcpyAsync(fit_host + c, h->d_hfit[b], m * 8, cudaMemcpyDeviceToHost, h->hs[b]));
    }
    CU(cudaStreamSynchronize(h->hs[0]));
    CU(cudaStreamSynchronize(h->hs[1]));
    return SPLIT_OK;
}

// ------------------------------------------------------------------------
// a1, a3-a9: the GA driver
// ------------------------------------------------------------------------
struct RunFlags {
    uint32_t export_end = 0, after_import = 0, init_gstall = 0;
};

static int run_kernel(split_ga_t* h, uint32_t mode, uint32_t g0, uint32_t g1, RunFlags fl = RunFlags{})
{
    GaArgs a = h->ga;
    a.mode = mode;
    a.trace = (mode == MODE_RUN) ? h->d_trace : nullptr;
    a.trace_gens = h->trace_gens;
    a.g_begin = g0;
    a.g_end = g1;
    a.export_end = fl.export_end;
    a.after_import = fl.after_import;
    a.init_gstall = fl.init_gstall;
    cudaError_t e = launch_ga(a, h->grid, h->stream, &h->stats.launches);
    if (e != cudaSuccess) return fail(SPLIT_E_CUDA, "GA kernel (mode %u): %s", mode, cudaGetErrorString(e));
    return SPLIT_OK;
}

static bool rec_better(double fa, const uint64_t* a, double fb, const uint64_t* b, uint32_t W)
{
    if (fa != fb) return fa > fb;
    for (int w = (int)W - 1; w >= 0; --w)
        if (a[w] != b[w]) return a[w] < b[w];
    return false;
}

// all-gather the exchange blocks in place: rank r contributes its islands' blocks at offset r * I blocks
static int allgather_xch(split_ga_t* h)
{
    SplitComm* c = (SplitComm*)h->p.comm;
    if (!c) return SPLIT_OK;                 // every island on this device: the blocks are already complete
    NcclApi* api = nccl_api();
    if (!api) return fail(SPLIT_E_NCCL, "NCCL not loadable");
    const size_t bytes = (size_t)h->ga.I * h->ga.xstride * 8;
    const char* src = (const char*)h->ga.xch + (size_t)c->rank * bytes;
    ncclResult_t r = api->allGather(src, h->ga.xch, bytes, ncclUint8, c->comm, h->stream);
    if (r != ncclSuccess) return fail(SPLIT_E_NCCL, "ncclAllGather: %s", api->getErrorString(r));
    return SPLIT_OK;
}

struct GlobalRec {
    double f;
    uint32_t gen;
    std::vector<uint64_t> bits;
};

// global best (R19) from the island records in the exchange blocks (host copy)
static void global_record(split_ga_t* h, const std::vector<uint64_t>& xch, GlobalRec* best)
{
    const uint32_t W = h->W, K = h->ga.K, It = h->ga.I_total;
    const size_t X = h->ga.xstride;
    bool have = false;
    const uint32_t first = h->p.comm ? 0 : h->ga.island_base;
    const uint32_t last = h->p.comm ? It : h->ga.island_base + h->ga.I;
    for (uint32_t g = first; g < last; ++g) {
        const uint64_t* e = xch.data() + (size_t)g * X + (size_t)K * W + K;
        double f;
        memcpy(&f, e, 8);
        const uint32_t gen = (uint32_t)(e[1] & 0xFFFFFFFFu);
        const uint64_t* bits = e + 2;
        if (!have || rec_better(f, bits, best->f, best->bits.data(), W) ||
            (f == best->f && memcmp(bits, best->bits.data(), W * 8) == 0 && gen < best->gen)) {
            best->f = f;
            best->gen = gen;
            best->bits.assign(bits, bits + W);
            have = true;
        }
    }
}

// Island segments are enqueued back to back with no host synchronisation: at a sync point g
// (g % M == 0, g < G) the RUN segment ends with the elite step of g, its K worst slots and each
// island's exchange block (top-K migrants + record); one ncclAllGather moves every block; the
// next segment's head applies the stall rule (ctl->done stops every later launch), places the
// foreign migrants and merges them into g's elites, then breeds.
extern "C" int split_ga_run(split_ga_t* h, uint32_t generations, uint64_t seed, split_best_t* best_out)
{
    if (!h || !best_out) return fail(SPLIT_E_INVAL, "split_ga_run: NULL argument");
    CU(cudaSetDevice(h->device));
    GaArgs& a = h->ga;
    a.key0 = (uint32_t)seed;
    a.key1 = (uint32_t)(seed >> 32);
    const bool single = a.I_total == 1;
    a.stall_in_kernel = single ? 1u : 0u;
    h->stats = split_run_stats{};
    CU(cudaMemsetAsync(a.rec_valid, 0, a.I * 4, h->stream));
    CU(cudaMemsetAsync(a.cand_cnt, 0, 3 * (size_t)a.I * a.cpi_pad * 4, h->stream));
    CU(cudaMemsetAsync(a.rc_cnt, 0, 3 * a.I * 4, h->stream));
    CU(cudaMemsetAsync(a.sel_cnt, 0, a.I * 4, h->stream));
    CU(cudaMemsetAsync(a.ghist, 0, 3 * a.I * 256 * 4, h->stream));
    CU(cudaMemsetAsync(a.tau, 0xFF, 2 * a.I * 8, h->stream));
    CU(cudaEventRecord(h->ev[0], h->stream));
    int rc = run_kernel(h, MODE_INIT, 0, 0);
    if (rc) return rc;
    CU(cudaEventRecord(h->ev[1], h->stream));
    const uint32_t M = h->p.migration_interval;
    const bool islands = !single && M > 0;
    if (!islands) {
        if (generations > 0) {
            rc = run_kernel(h, MODE_RUN, 0, generations);
            if (rc) return rc;
        }
    } else {
        rc = allgather_xch(h);                        // generation-0 records: the global stall baseline
        if (rc) return rc;
        uint32_t g = 0;
        while (g < generations) {
            const uint32_t g1 = std::min<uint32_t>((g / M + 1) * M, generations);
            RunFlags fl;
            fl.export_end = (g1 % M == 0 && g1 < generations) ? 1u : 0u;
            fl.after_import = g > 0 ? 1u : 0u;
            fl.init_gstall = g == 0 ? 1u : 0u;
            rc = run_kernel(h, MODE_RUN, g, g1, fl);
            if (rc) return rc;
            if (!fl.export_end) break;
            rc = allgather_xch(h);                    // the next segment's head imports from the blocks
            if (rc) return rc;
            g = g1;
        }
    }
    CU(cudaEventRecord(h->ev[2], h->stream));
    rc = allgather_xch(h);                            // final records (the last launch packed them)
    if (rc) return rc;
    Ctl ctl;
    std::vector<uint64_t> xh((size_t)a.I_total * a.xstride);
    CU(cudaMemcpyAsync(&ctl, a.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, h->stream));
    CU(cudaMemcpyAsync(xh.data(), a.xch, xh.size() * 8, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    const uint32_t gens_run = generations > 0 ? ctl.gens_run : 0;
    h->stats.general_selects = ctl.n_general;
    h->stats.fast_selects = ctl.n_fast;
    GlobalRec best;
    global_record(h, xh, &best);
    // statistics of the best split
    CU(cudaMemcpyAsync(h->d_bits1, best.bits.data(), h->W * 8, cudaMemcpyHostToDevice, h->stream));
    CU(launch_eval_stats(h->ch, h->d_bits1, h->d_stats, h->d_statf, h->stream));
    ++h->stats.launches;
    int64_t st[5];
    double fchk;
    CU(cudaMemcpyAsync(st, h->d_stats, sizeof(st), cudaMemcpyDeviceToHost, h->stream));
    CU(cudaMemcpyAsync(&fchk, h->d_statf, 8, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    CU(cudaEventElapsedTime(&h->stats.ms_total, h->ev[0], h->ev[2]));
    CU(cudaEventElapsedTime(&h->stats.ms_loop, h->ev[1], h->ev[2]));
    if (best_out->bits) memcpy(best_out->bits, best.bits.data(), h->W * 8);
    best_out->fitness = best.f;
    best_out->k = (uint32_t)st[0];
    best_out->var_num = st[1];
    best_out->s1 = (uint64_t)st[2];
    best_out->s2 = (uint64_t)st[3];
    best_out->overhead_ns = (uint64_t)st[4];
    best_out->expected_wait_ns = st[2] > 0 ? (double)(uint64_t)st[3] / (2.0 * (double)(uint64_t)st[2]) : 0.0;
    best_out->generation_found = best.gen;
    best_out->generations_run = gens_run;
    best_out->evaluations = (uint64_t)a.I * ((uint64_t)a.N + (uint64_t)gens_run * (a.N - a.E));
    h->last_gen = gens_run;
    h->have_pop = true;
    if (h->d_trace) {
        std::vector<unsigned long long> tr((size_t)h->trace_gens * 16 + kTraceArrGens * 1024);
        CU(cudaMemcpy(tr.data(), h->d_trace, tr.size() * 8, cudaMemcpyDeviceToHost));
        if (FILE* f = fopen(getenv("SPLIT_TRACE"), "w")) {
            fprintf(f, "gen,lead_start,lead_record,lead_sort,lead_end,work_start,work_end,lead_sync,work_sync,"
                       "b_tourn,b_rows,b_repair,b_eval,b_rec,b_xover,b_cand,lead_loaded\n");
            CU(cudaMemset(h->d_trace, 0, tr.size() * 8));
            for (uint32_t g = 0; g < h->trace_gens; ++g) {
                fprintf(f, "%u", g);
                for (int j = 0; j < 16; ++j) fprintf(f, ",%llu", tr[(size_t)g * 16 + j]);
                fprintf(f, "\n");
            }
            fclose(f);
            // per-CTA arrival instants of kTraceArrGens generations: <path>.arrivals
            std::string p2 = std::string(getenv("SPLIT_TRACE")) + ".arrivals";
            if (FILE* f2 = fopen(p2.c_str(), "w")) {
                for (uint32_t g = 0; g < kTraceArrGens; ++g) {
                    fprintf(f2, "%u", g);
                    for (int c = 0; c < h->grid; ++c) fprintf(f2, ",%llu", tr[(size_t)h->trace_gens * 16 + g * 1024 + c]);
                    fprintf(f2, "\n");
                }
                fclose(f2);
            }
        }
    }
    if (fchk != best.f) return fail(SPLIT_E_STATE, "best record fitness mismatch (internal)");
    return SPLIT_OK;
}

extern "C" int split_ga_population(split_ga_t* h, uint32_t island, uint64_t* bits_host, double* fit_host)
{
    if (!h) return fail(SPLIT_E_INVAL, "split_ga_population: NULL handle");
    if (!h->have_pop) return fail(SPLIT_E_STATE, "no population: call split_ga_run first");
    if (island >= h->ga.I) return fail(SPLIT_E_INVAL, "local island out of range");
    CU(cudaSetDevice(h->device));
    const uint32_t b = h->last_gen & 1u;
    const size_t N = h->ga.N, W = h->W;
    if (bits_host)
        CU(cudaMemcpyAsync(bits_host, h->ga.pop[b] + island * N * W, N * W * 8, cudaMemcpyDeviceToHost, h->stream));
    if (fit_host)
        CU(cudaMemcpyAsync(fit_host, h->ga.fit[b] + island * (size_t)h->ga.Ns, N * 8, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    return SPLIT_OK;
}

extern "C" int split_last_run_stats(const split_ga_t* h, split_run_stats* out)
{
    if (!h || !out) return fail(SPLIT_E_INVAL, "NULL argument");
    *out = h->stats;
    return SPLIT_OK;
}

// ------------------------------------------------------------------------
// a10 — Algorithm 1 (greedy preemption), reading R12:
// scanning from the tail, t_new passes t_i iff the types differ and
// Ext_left(t_i)*Ext(t_i) > Ext_left(t_new)*Ext(t_new); it stops behind the
// first t_i it does not pass, or reaches the head.  alpha and the waited
// times cancel out of line 13's comparison.
// ------------------------------------------------------------------------
static bool req_ok(const split_request& r) { return r.ext_ns > 0 && r.ext_left_ns >= 0 && r.ext_left_ns <= r.ext_ns; }

extern "C" int split_preempt_decide(const split_queue_state* q, uint32_t* insert_pos)
{
    if (!q || !insert_pos) return fail(SPLIT_E_INVAL, "split_preempt_decide: NULL argument");
    if (!(q->alpha > 0.0) || !isfinite(q->alpha)) return fail(SPLIT_E_INVAL, "alpha must be > 0");
    if (q->n > 0 && !q->queue) return fail(SPLIT_E_INVAL, "queue is NULL");
    if (!req_ok(q->incoming)) return fail(SPLIT_E_INVAL, "incoming request: need ext > 0, 0 <= ext_left <= ext");
    for (uint32_t i = 0; i < q->n; ++i)
        if (!req_ok(q->queue[i])) return fail(SPLIT_E_INVAL, "queue[%u]: need ext > 0, 0 <= ext_left <= ext", i);
    const __int128 w_new = (__int128)q->incoming.ext_left_ns * q->incoming.ext_ns;
    for (uint32_t j = q->n; j-- > 0;) {
        const split_request& t = q->queue[j];
        if (t.type_id == q->incoming.type_id) { *insert_pos = j + 1; return SPLIT_OK; }
        if ((__int128)t.ext_left_ns * t.ext_ns <= w_new) { *insert_pos = j + 1; return SPLIT_OK; }
    }
    *insert_pos = 0;
    return SPLIT_OK;
}

// ------------------------------------------------------------------------
// block times of a split (host; R2, R3): the block after cut p pays ovh[p]
// ------------------------------------------------------------------------
extern "C" int split_block_times(const int64_t* lat, const int64_t* ovh, uint32_t n, const uint64_t* bits,
                                 int64_t* out_ns, uint32_t cap, uint32_t* k)
{
    if (!lat || !bits || !k || (cap > 0 && !out_ns)) return fail(SPLIT_E_INVAL, "split_block_times: NULL argument");
    if (n < 2) return fail(SPLIT_E_INVAL, "split_block_times: n_ops must be >= 2");
    for (uint32_t i = 0; i < n; ++i)
        if (lat[i] < 0) return fail(SPLIT_E_INVAL, "latencies_ns[%u] < 0", i);
    if (ovh)
        for (uint32_t i = 0; i + 1 < n; ++i)
            if (ovh[i] < 0) return fail(SPLIT_E_INVAL, "cut_overhead_ns[%u] < 0", i);
    uint32_t j = 0;
    int64_t cur = 0;
    for (uint32_t p = 0; p < n; ++p) {
        cur += lat[p];
        const bool cut = p + 1 < n && ((bits[p >> 6] >> (p & 63)) & 1ull);
        if (cut || p + 1 == n) {
            if (j < cap) out_ns[j] = cur;
            ++j;
            cur = cut ? (ovh ? ovh[p] : 0) : 0;
        }
    }
    *k = j;
    if (j > cap) return fail(SPLIT_E_RANGE, "split_block_times: %u blocks > cap %u", j, cap);
    return SPLIT_OK;
}

// ------------------------------------------------------------------------
// device self-tests
// ------------------------------------------------------------------------
extern "C" int split_selftest_philox(int device, const uint32_t* in, uint32_t n, uint32_t* out)
{
    if ((!in || !out) && n) return fail(SPLIT_E_INVAL, "NULL buffer");
    if (n == 0) return SPLIT_OK;
    CU(cudaSetDevice(device));
    uint32_t *di = nullptr, *dout = nullptr;
    CU(cudaMalloc(&di, (size_t)n * 24));
    CU(cudaMalloc(&dout, (size_t)n * 16));
    cudaError_t e = cudaMemcpy(di, in, (size_t)n * 24, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = launch_selftest_philox(di, n, dout, 0);
    if (e == cudaSuccess) e = cudaMemcpy(out, dout, (size_t)n * 16, cudaMemcpyDeviceToHost);
    cudaFree(di);
    cudaFree(dout);
    if (e != cudaSuccess) return fail(SPLIT_E_CUDA, "selftest_philox: %s", cudaGetErrorString(e));
    return SPLIT_OK;
}

extern "C" int split_selftest_dexp(int device, const double* in, uint32_t n, double* out)
{
    if ((!in || !out) && n) return fail(SPLIT_E_INVAL, "NULL buffer");
    if (n == 0) return SPLIT_OK;
    CU(cudaSetDevice(device));
    double *di = nullptr, *dout = nullptr;
    CU(cudaMalloc(&di, (size_t)n * 8));
    CU(cudaMalloc(&dout, (size_t)n * 8));
    cudaError_t e = cudaMemcpy(di, in, (size_t)n * 8, cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = launch_selftest_dexp(di, n, dout, 0);
    if (e == cudaSuccess) e = cudaMemcpy(out, dout, (size_t)n * 8, cudaMemcpyDeviceToHost);
    cudaFree(di);
    cudaFree(dout);
    if (e != cudaSuccess) return fail(SPLIT_E_CUDA, "selftest_dexp: %s", cudaGetErrorString(e));
    return SPLIT_OK;
}

// ------------------------------------------------------------------------
// f1 exact solvers: exhaustive enumeration and the DP
// ------------------------------------------------------------------------
#define RC(x)                      \
    do {                            \
        const int rc_ = (x);        \
        if (rc_ != SPLIT_OK) return rc_; \
    } while (0)

namespace {
// scratch owned by one call (freed on every exit path)
struct DevScratch {
    std::vector<void*> p;
    ~DevScratch()
    {
        for (void* q : p) cudaFree(q);
    }
    template <class T>
    int alloc(T** out, size_t count)
    {
        void* q = nullptr;
        cudaError_t e = cudaMalloc(&q, count * sizeof(T) + 16);
        if (e != cudaSuccess) return fail(SPLIT_E_NOMEM, "cudaMalloc(%zu): %s", count * sizeof(T), cudaGetErrorString(e));
        p.push_back(q);
        *out = (T*)q;
        return SPLIT_OK;
    }
};
}  // namespace

extern "C" int split_exhaustive(split_ga_t* h, split_best_t* best_out, int64_t* min_v_per_k, uint64_t* argmin_per_k)
{
    if (!h || !best_out || !best_out->bits) return fail(SPLIT_E_INVAL, "split_exhaustive: NULL argument");
    const uint32_t m = h->n - 1;
    if (m > kExhMaxPos) return fail(SPLIT_E_INVAL, "split_exhaustive: n_ops - 1 = %u cut positions > %u", m, kExhMaxPos);
    if (h->p.k_max > 64) return fail(SPLIT_E_INVAL, "split_exhaustive: k_max must be <= 64");
    CU(cudaSetDevice(h->device));
    const uint32_t c = m < kExhLow ? m : kExhLow;
    // A[p] = P[p+1] (A[m] = T), B[p] = P[p+1] - ovh[p] (mod 2^32)
    std::vector<uint32_t> A(m + 1), B(m > 0 ? m : 1);
    for (uint32_t q = 0; q <= m; ++q) A[q] = h->hwords[q + 1];
    for (uint32_t q = 0; q < m; ++q) B[q] = h->hwords[q + 1] - h->hwords[h->p_words + q];
    DevScratch sc;
    uint32_t *dA, *dB;
    void *dtab, *dres, *dout;
    uint64_t *dkv, *dkv2;
    const size_t rows = m - c + 1, nb = (size_t)1 << c;
    RC(sc.alloc(&dA, A.size()));
    RC(sc.alloc(&dB, B.size()));
    RC(sc.alloc((uint8_t**)&dtab, rows * nb * 16));
    RC(sc.alloc(&dkv, 65));
    RC(sc.alloc(&dkv2, 65));
    CU(cudaMemcpyAsync(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice, h->stream));
    CU(cudaMemcpyAsync(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice, h->stream));
    ExhArgs a;
    memset(&a, 0, sizeof(a));
    a.A = dA;
    a.B = dB;
    a.tab = dtab;
    a.m = m;
    a.c = c;
    a.T = (uint32_t)h->T;
    a.rcp = h->ch.rcp;
    a.k_min = h->p.k_min;
    a.k_max = h->p.k_max;
    a.outer_total = (uint64_t)1 << (m - c);
    a.seed_f = 0.0;
    // grid: enough threads to fill every SM, each walking a contiguous Gray range
    const uint64_t max_threads = (uint64_t)exh_blocks_per_sm(a) * h->num_sms * kExhThreads;
    uint64_t threads = a.outer_total < max_threads ? a.outer_total : max_threads;
    a.per_thread = (a.outer_total + threads - 1) / threads;
    threads = (a.outer_total + a.per_thread - 1) / a.per_thread;
    const uint32_t grid = (uint32_t)((threads + kExhThreads - 1) / kExhThreads);
    RC(sc.alloc((uint8_t**)&dres, (size_t)grid * 16));
    RC(sc.alloc((uint8_t**)&dout, 16));
    a.res = dres;
    h->stats.launches = 0;
    CU(launch_exh_table(a, h->stream));
    ++h->stats.launches;
    CU(cudaEventRecord(h->ev[0], h->stream));
    CU(launch_exh(a, MODE_EXH_BEST, grid, h->stream));
    CU(launch_exh_reduce(dres, grid, dout, h->stream));
    CU(cudaEventRecord(h->ev[2], h->stream));
    h->stats.launches += 2;
    struct {
        double f;
        uint64_t bits;
    } best;
    CU(cudaMemcpyAsync(&best, dout, 16, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    CU(cudaEventElapsedTime(&h->stats.ms_total, h->ev[0], h->ev[2]));
    h->stats.ms_loop = h->stats.ms_total;
    if (best.f == -INFINITY) return fail(SPLIT_E_STATE, "split_exhaustive: no split with k in [k_min, k_max]");
    // statistics of the best split (same kernel as split_ga_run's)
    CU(cudaMemcpyAsync(h->d_bits1, &best.bits, 8, cudaMemcpyHostToDevice, h->stream));
    CU(launch_eval_stats(h->ch, h->d_bits1, h->d_stats, h->d_statf, h->stream));
    ++h->stats.launches;
    int64_t st[5];
    double fchk;
    CU(cudaMemcpyAsync(st, h->d_stats, sizeof(st), cudaMemcpyDeviceToHost, h->stream));
    CU(cudaMemcpyAsync(&fchk, h->d_statf, 8, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    if (fchk != best.f) return fail(SPLIT_E_STATE, "split_exhaustive: best fitness mismatch (internal)");
    best_out->bits[0] = best.bits;
    for (uint32_t w = 1; w < h->W; ++w) best_out->bits[w] = 0;
    best_out->fitness = best.f;
    best_out->k = (uint32_t)st[0];
    best_out->var_num = st[1];
    best_out->s1 = (uint64_t)st[2];
    best_out->s2 = (uint64_t)st[3];
    best_out->overhead_ns = (uint64_t)st[4];
    best_out->expected_wait_ns = st[2] > 0 ? (double)(uint64_t)st[3] / (2.0 * (double)(uint64_t)st[2]) : 0.0;
    best_out->generation_found = 0;
    best_out->generations_run = 0;
    best_out->evaluations = (uint64_t)1 << m;
    if (min_v_per_k || argmin_per_k) {
        // MINV pass: min V per k <= k_max; ARGMIN pass: smallest bitset attaining it
        std::vector<uint64_t> init(65, ~0ull), kv(65), kb(65);
        CU(cudaMemcpyAsync(dkv, init.data(), 65 * 8, cudaMemcpyHostToDevice, h->stream));
        a.kv_out = dkv;
        CU(launch_exh(a, MODE_EXH_MINV, grid, h->stream));
        ++h->stats.launches;
        CU(cudaMemcpyAsync(kv.data(), dkv, 65 * 8, cudaMemcpyDeviceToHost, h->stream));
        if (argmin_per_k) {
            CU(cudaMemcpyAsync(dkv2, init.data(), 65 * 8, cudaMemcpyHostToDevice, h->stream));
            a.kv = dkv;
            a.kv_out = dkv2;
            CU(launch_exh(a, MODE_EXH_ARGMIN, grid, h->stream));
            ++h->stats.launches;
            CU(cudaMemcpyAsync(kb.data(), dkv2, 65 * 8, cudaMemcpyDeviceToHost, h->stream));
        }
        CU(cudaStreamSynchronize(h->stream));
        for (uint32_t k = 0; k <= h->p.k_max; ++k) {
            if (min_v_per_k) min_v_per_k[k] = (kv[k] == ~0ull) ? -1 : (int64_t)kv[k];
            if (argmin_per_k) argmin_per_k[k] = (kv[k] == ~0ull) ? 0 : kb[k];
        }
    }
    return SPLIT_OK;
}

extern "C" int split_heatmap2(split_ga_t* h, int64_t* var_out, uint64_t* ov_out, double* fit_out)
{
    if (!h) return fail(SPLIT_E_INVAL, "split_heatmap2: NULL handle");
    if (h->p.k_max < 3 && h->n > 2)
        return fail(SPLIT_E_INVAL, "split_heatmap2: the handle's k_max must be >= 3 (its guards cover two cuts)");
    if (((uintptr_t)var_out | (uintptr_t)ov_out | (uintptr_t)fit_out) & 7u)
        return fail(SPLIT_E_ALIGN, "split_heatmap2: outputs must be 8-byte aligned");
    if (!var_out && !ov_out && !fit_out) return SPLIT_OK;
    CU(cudaSetDevice(h->device));
    CU(launch_heatmap2(h->ch, var_out, ov_out, fit_out, h->stream));
    h->stats.launches = 1;
    return SPLIT_OK;
}

extern "C" int split_dp_min_s2(split_ga_t* h, uint32_t k_max, uint64_t* s2_out)
{
    if (!h || !s2_out) return fail(SPLIT_E_INVAL, "split_dp_min_s2: NULL argument");
    if (k_max < 1 || k_max > h->p.k_max)
        return fail(SPLIT_E_INVAL, "split_dp_min_s2: k_max must be in [1, handle k_max = %u]", h->p.k_max);
    CU(cudaSetDevice(h->device));
    DevScratch sc;
    uint64_t* d_out;
    RC(sc.alloc(&d_out, (size_t)k_max + 1));
    CU(cudaEventRecord(h->ev[0], h->stream));
    CU(launch_dp(h->ch.words, h->ch.words + h->ch.p_words, h->n, k_max, d_out, h->stream));
    CU(cudaEventRecord(h->ev[2], h->stream));
    h->stats.launches = 1;
    CU(cudaMemcpyAsync(s2_out, d_out, ((size_t)k_max + 1) * 8, cudaMemcpyDeviceToHost, h->stream));
    CU(cudaStreamSynchronize(h->stream));
    CU(cudaEventElapsedTime(&h->stats.ms_total, h->ev[0], h->ev[2]));
    h->stats.ms_loop = h->stats.ms_total;
    return SPLIT_OK;
}

// ------------------------------------------------------------------------
// f2: QoS simulator (split_qos.cu)
// ------------------------------------------------------------------------
static int qos_simulate(const int64_t* blocks_ns, const uint32_t* n_blocks, uint32_t n_types, uint32_t policy,
                        const int64_t* unsplit_ns, const int64_t* ref_ns, uint32_t d_max, uint32_t s_max,
                        const uint32_t* alpha_milli,
                        uint32_t n_alpha, uint64_t n_rep, uint32_t n_req, const int64_t* arrival_ns,
                        const uint32_t* type_id, int64_t* t_ete_out, uint32_t* viol_out, double* rr_out, int device,
                        void* stream)
{
    if (!blocks_ns || !n_blocks || n_types == 0 || n_types > 65535)
        return fail(SPLIT_E_INVAL, "split_qos_simulate: need 1..65535 model types with their blocks");
    if (policy > 2 || (policy == 2) != (unsplit_ns != nullptr))
        return fail(SPLIT_E_INVAL, "split_qos_simulate: policy must be 0 (FIFO) or 1 (Algorithm 1); elastic needs unsplit_ns");
    std::vector<uint32_t> uns;
    if (policy == 2)
        for (uint32_t m = 0; m < n_types; ++m) {
            if (unsplit_ns[m] < 1 || unsplit_ns[m] >= ((int64_t)1 << 32))
                return fail(SPLIT_E_RANGE, "split_qos_simulate_elastic: unsplit time out of [1, 2^32)");
            uns.push_back((uint32_t)unsplit_ns[m]);
        }
    std::vector<uint32_t> refv;
    if (ref_ns)
        for (uint32_t m = 0; m < n_types; ++m) {
            if (ref_ns[m] < 1 || ref_ns[m] >= ((int64_t)1 << 32))
                return fail(SPLIT_E_RANGE, "split_qos_simulate_elastic: ref_ns out of [1, 2^32)");
            refv.push_back((uint32_t)ref_ns[m]);
        }
    if (n_alpha > kQosMaxAlpha || (n_alpha && !alpha_milli))
        return fail(SPLIT_E_INVAL, "split_qos_simulate: at most %u alpha thresholds", kQosMaxAlpha);
    if (n_rep == 0 || n_req == 0) return SPLIT_OK;
    if (!arrival_ns || !type_id || !t_ete_out || !rr_out || (n_alpha && !viol_out))
        return fail(SPLIT_E_INVAL, "split_qos_simulate: NULL device buffer");
    std::vector<uint32_t> off(n_types + 1, 0), ext(n_types, 0), blk;
    for (uint32_t m = 0; m < n_types; ++m) {
        if (n_blocks[m] == 0 || n_blocks[m] > 65535)
            return fail(SPLIT_E_INVAL, "split_qos_simulate: model %u has %u blocks (need 1..65535)", m, n_blocks[m]);
        uint64_t e = 0;
        for (uint32_t j = 0; j < n_blocks[m]; ++j) {
            const int64_t b = blocks_ns[off[m] + j];
            if (b < 1 || b >= ((int64_t)1 << 32)) return fail(SPLIT_E_RANGE, "split_qos_simulate: block time out of [1, 2^32)");
            e += (uint64_t)b;
            blk.push_back((uint32_t)b);
        }
        if (e >= ((uint64_t)1 << 32)) return fail(SPLIT_E_RANGE, "split_qos_simulate: Ext(model %u) >= 2^32 ns", m);
        ext[m] = (uint32_t)e;
        off[m + 1] = off[m] + n_blocks[m];
    }
    for (uint32_t j = 0; j < n_alpha; ++j)
        if (alpha_milli[j] == 0) return fail(SPLIT_E_INVAL, "split_qos_simulate: alpha must be > 0");
    CU(cudaSetDevice(device));
    cudaStream_t st = (cudaStream_t)stream;
    std::vector<uint32_t> tab;
    tab.insert(tab.end(), off.begin(), off.end());
    tab.insert(tab.end(), ext.begin(), ext.end());
    tab.insert(tab.end(), alpha_milli, alpha_milli + n_alpha);
    tab.insert(tab.end(), blk.begin(), blk.end());
    tab.insert(tab.end(), uns.begin(), uns.end());
    if (refv.empty()) refv = ext;                       // statistics against the split model's Ext (R20)
    tab.insert(tab.end(), refv.begin(), refv.end());
    tab.push_back(0);                                   // error flag
    QosArgs a;
    memset(&a, 0, sizeof(a));
    a.n_types = n_types;
    a.n_blocks_total = (uint32_t)blk.size();
    a.n_alpha = n_alpha;
    a.policy = policy;
    a.n_rep = n_rep;
    a.n_req = n_req;
    a.arrival = arrival_ns;
    a.type = type_id;
    a.t_ete = t_ete_out;
    a.viol = viol_out;
    a.rr = rr_out;
    a.d_max = d_max;
    a.s_max = s_max;
    if (qos_smem_bytes(a, kQosQueueBig) > 227 * 1024) return fail(SPLIT_E_INVAL, "split_qos_simulate: model tables too large");
    // stream-ordered scratch (no device-wide synchronisation in cudaFree)
    uint32_t* d_tab = nullptr;
    CU(cudaMallocAsync((void**)&d_tab, tab.size() * 4, st));
    struct FreeAsync {
        void* p;
        cudaStream_t s;
        ~FreeAsync() { cudaFreeAsync(p, s); }
    } guard{d_tab, st};
    CU(cudaMemcpyAsync(d_tab, tab.data(), tab.size() * 4, cudaMemcpyHostToDevice, st));
    a.blk_off = d_tab;
    a.ext = d_tab + n_types + 1;
    a.alpha_milli = a.ext + n_types;
    a.blk_ns = a.alpha_milli + n_alpha;
    a.uns = a.blk_ns + blk.size();
    a.ref = a.uns + uns.size();
    a.err = d_tab + tab.size() - 1;
    CU(launch_qos(a, st, kQosQueue));
    uint32_t err = 0;
    CU(cudaMemcpyAsync(&err, a.err, 4, cudaMemcpyDeviceToHost, st));
    CU(cudaStreamSynchronize(st));
    if (err == 2) {
        // some replica held more than kQosQueue pending requests (an overloaded system): the whole batch
        // again with the large queue (fewer replicas per SM; every output is rewritten)
        CU(cudaMemsetAsync(a.err, 0, 4, st));
        CU(launch_qos(a, st, kQosQueueBig));
        CU(cudaMemcpyAsync(&err, a.err, 4, cudaMemcpyDeviceToHost, st));
        CU(cudaStreamSynchronize(st));
    }
    if (err == 1) return fail(SPLIT_E_RANGE, "split_qos_simulate: arrivals not non-decreasing / negative, or type id >= n_types");
    if (err == 2) return fail(SPLIT_E_RANGE, "split_qos_simulate: more than %u pending requests (overloaded)", kQosQueueBig);
    return SPLIT_OK;
}

extern "C" int split_qos_simulate(const int64_t* blocks_ns, const uint32_t* n_blocks, uint32_t n_types, uint32_t policy,
                                  const uint32_t* alpha_milli, uint32_t n_alpha, uint64_t n_rep, uint32_t n_req,
                                  const int64_t* arrival_ns, const uint32_t* type_id, int64_t* t_ete_out,
                                  uint32_t* viol_out, double* rr_out, int device, void* stream)
{
    if (policy > 1) return fail(SPLIT_E_INVAL, "split_qos_simulate: policy must be 0 (FIFO) or 1 (Algorithm 1)");
    return qos_simulate(blocks_ns, n_blocks, n_types, policy, nullptr, nullptr, 0, 0, alpha_milli, n_alpha, n_rep, n_req,
                        arrival_ns, type_id, t_ete_out, viol_out, rr_out, device, stream);
}

extern "C" int split_qos_simulate_elastic(const int64_t* blocks_ns, const uint32_t* n_blocks, const int64_t* unsplit_ns,
                                          const int64_t* ref_ns, uint32_t n_types, uint32_t d_max, uint32_t s_max,
                                          const uint32_t* alpha_milli, uint32_t n_alpha, uint64_t n_rep,
                                          uint32_t n_req, const int64_t* arrival_ns, const uint32_t* type_id,
                                          int64_t* t_ete_out, uint32_t* viol_out, double* rr_out, int device,
                                          void* stream)
{
    if (!unsplit_ns) return fail(SPLIT_E_INVAL, "split_qos_simulate_elastic: NULL unsplit_ns");
    return qos_simulate(blocks_ns, n_blocks, n_types, 2, unsplit_ns, ref_ns, d_max, s_max, alpha_milli, n_alpha, n_rep, n_req,
                        arrival_ns, type_id, t_ete_out, viol_out, rr_out, device, stream);
}
