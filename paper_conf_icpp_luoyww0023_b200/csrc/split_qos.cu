// split_qos.cu — f2: batched Monte-Carlo of SPLIT's request scheduling
// (ICPP'23 §3.4 Algorithm 1 over split models, §5 QoS metrics).
//
// One thread simulates one replica: an edge executor serving n_req requests of
// n_types split models, preempting only between blocks (P@24400-26700), the
// queue order decided at each arrival by Algorithm 1 under reading R12 (pass
// t_i iff its type differs and Ext_left(t_i) Ext(t_i) > Ext_left(new) Ext(new))
// or FIFO.  Event semantics: DESIGN.md R20.  Everything is exact integer ns;
// the two sums of response ratios (Eq. 3) are IEEE doubles added in request
// order, so results are bit-identical to oracle/qos.py.
//
// Layout: request streams are request-major (element [i][r] of replica r at
// i * n_rep + r), so a warp's loads and stores of request i are coalesced; the
// pending queue of each thread lives in shared memory in SoA form
// q[j][tid] (entry j of thread tid at j * kQosThreads + tid: conflict-free),
// the model tables (block offsets, block ns, Ext per type) and the alpha list
// are staged once per CTA.
#include "split_device.cuh"

namespace splitga {

// kConverge: advance every replica of a warp by one event per loop trip and re-converge the warp
// after it (policy 2; see the loop).  Policies 0/1 run the free-running loop, measured faster there.
template <bool kConverge, uint32_t QCAP>
__global__ void __launch_bounds__(kQosThreads) qos_kernel(QosArgs a)
{
    extern __shared__ __align__(16) uint8_t smem[];
    uint32_t* s_off = (uint32_t*)smem;                    // [M + 1]
    uint32_t* s_ext = s_off + a.n_types + 1;              // [M]
    uint32_t* s_alpha = s_ext + a.n_types;                // [n_alpha]
    uint32_t* s_blk = s_alpha + a.n_alpha;                // [total blocks]
    const uint32_t nb = a.n_blocks_total;
    uint32_t* q_req = s_blk + nb;                         // [QCAP][kQosThreads]
    uint32_t* q_left = q_req + QCAP * kQosThreads;        // Ext_left (ns)
    uint32_t* q_tb = q_left + QCAP * kQosThreads;         // type | next block << 16
    uint32_t* s_viol = q_tb + QCAP * kQosThreads;         // [n_alpha][kQosThreads]
    uint32_t* s_uns = s_viol + a.n_alpha * kQosThreads;   // [M] unsplit T (policy 2)
    uint32_t* s_ref = s_uns + a.n_types;                  // [M] latency reference of the statistics
    for (uint32_t j = threadIdx.x; j <= a.n_types; j += blockDim.x) s_off[j] = a.blk_off[j];
    for (uint32_t j = threadIdx.x; j < a.n_types; j += blockDim.x) s_ext[j] = a.ext[j];
    for (uint32_t j = threadIdx.x; j < a.n_alpha; j += blockDim.x) s_alpha[j] = a.alpha_milli[j];
    for (uint32_t j = threadIdx.x; j < nb; j += blockDim.x) s_blk[j] = a.blk_ns[j];
    if (a.policy == 2u)
        for (uint32_t j = threadIdx.x; j < a.n_types; j += blockDim.x) s_uns[j] = a.uns[j];
    for (uint32_t j = threadIdx.x; j < a.n_types; j += blockDim.x) s_ref[j] = a.ref[j];
    __syncthreads();
    const uint32_t tid = threadIdx.x;
    const uint64_t r = (uint64_t)blockIdx.x * blockDim.x + tid;
    if (r >= a.n_rep) return;
    const uint32_t n_req = a.n_req;
    const uint64_t st = a.n_rep;                          // request-major stride
    const int64_t* arr = a.arrival + r;
    const uint32_t* ty = a.type + r;
    int64_t* te = a.t_ete + r;
#define Q(arr_, j) arr_[(j) * kQosThreads + tid]
    uint32_t n = 0, i = 0, done = 0;
    bool idle = true, run_last = false;
    int64_t busy = 0, run_arr = 0, now = 0;
    uint32_t run_req = 0;
    int64_t next_a = n_req ? __ldcs(arr) : 0;
    uint32_t next_t = n_req ? __ldcs(ty) : 0;
    int64_t prev_a = 0;
    uint32_t err = 0;
    // lanes of this warp that hold a replica (the grid's last warp may be partial)
    const uint64_t wbase = r - (tid & 31u);
    const uint64_t nl = a.n_rep - wbase;
    const unsigned wmask = nl >= 32 ? 0xFFFFFFFFu : ((1u << nl) - 1u);
    // start the next block of the queue head (executor idle)
    auto dispatch = [&]() {
        if (!idle || n == 0) return;
        const uint32_t tb = Q(q_tb, 0), m = tb & 0xFFFFu, blk = tb >> 16;
        const uint32_t b = (blk == kQosUnsplit) ? s_uns[m] : s_blk[s_off[m] + blk];
        const uint32_t left = Q(q_left, 0) - b;
        run_req = Q(q_req, 0);
        busy = now + b;
        idle = false;
        run_last = (left == 0u);
        if (run_last) {
            run_arr = __ldg(arr + run_req * st);          // needed only when the request completes
            for (uint32_t j = 1; j < n; ++j) {
                Q(q_req, j - 1) = Q(q_req, j);
                Q(q_left, j - 1) = Q(q_left, j);
                Q(q_tb, j - 1) = Q(q_tb, j);
            }
            --n;
        } else {
            Q(q_left, 0) = left;
            Q(q_tb, 0) = tb + (1u << 16);
        }
    };
    // kConverge: one event per thread per warp-iteration, with the warp re-converged after each: the
    // replicas' event sequences differ, and under policy 2 the warp's threads otherwise drift apart and
    // issue their events one subset at a time (4x the warp instructions, DESIGN.md f4).
    bool live = done < n_req;
    while (kConverge ? __any_sync(wmask, live) : live) {
        if (live) {
            do {
                if (!idle && (i >= n_req || busy < next_a)) {
                    now = busy;                                   // block end
                    if (run_last) {
                        __stcs(te + run_req * st, now - run_arr);
                        ++done;
                    }
                    idle = true;
                    dispatch();
                } else {
                    now = next_a;                                 // arrival (first on ties)
                    if (now < prev_a || now < 0 || next_t >= a.n_types) { err = 1u; break; }
                    prev_a = now;
                    const uint32_t m = next_t, e = s_ext[m];
                    uint32_t pos = n, left0 = e, tb0 = m;
                    if (a.policy != 0u) {
                        // Algorithm 1 (R12): scan from the tail; stay behind the first request of
                        // the same type or with Ext_left * Ext <= Ext_left(new) * Ext(new)
                        const uint64_t key = (uint64_t)e * e;
                        pos = 0;
                        for (uint32_t j = n; j-- > 0;) {
                            const uint32_t tj = Q(q_tb, j) & 0xFFFFu;
                            if (tj == m || (uint64_t)Q(q_left, j) * s_ext[tj] <= key) { pos = j + 1; break; }
                        }
                    }
                    if (a.policy == 2u) {
                        // f4 elastic splitting (R23): suspended under high density or many requests of the
                        // same type -> unsplit, at the tail
                        uint32_t same = 0;
                        for (uint32_t j = 0; j < n; ++j) same += ((Q(q_tb, j) & 0xFFFFu) == m) ? 1u : 0u;
                        const bool off = (n >= a.d_max) | (same >= a.s_max);
                        pos = off ? n : pos;
                        left0 = off ? s_uns[m] : e;
                        tb0 = off ? (m | (kQosUnsplit << 16)) : m;
                    }
                    if (n == QCAP) { err = 2u; break; }
                    for (uint32_t j = n; j > pos; --j) {
                        Q(q_req, j) = Q(q_req, j - 1);
                        Q(q_left, j) = Q(q_left, j - 1);
                        Q(q_tb, j) = Q(q_tb, j - 1);
                    }
                    Q(q_req, pos) = i;
                    Q(q_left, pos) = left0;
                    Q(q_tb, pos) = tb0;
                    ++n;
                    ++i;
                    if (i < n_req) {
                        next_a = __ldcs(arr + i * st);
                        next_t = __ldcs(ty + i * st);
                    }
                    dispatch();
                }
            } while (0);
            live = (err == 0u) && (done < n_req);
        }
        if (kConverge) __syncwarp(wmask);
    }
#undef Q
    if (err) {
        atomicMax(a.err, err);
        return;
    }
    // statistics in request order (R20)
    for (uint32_t j = 0; j < a.n_alpha; ++j) s_viol[j * kQosThreads + tid] = 0;
    double rs = 0.0, rq = 0.0;
    for (uint32_t k = 0; k < n_req; ++k) {
        const int64_t t = __ldcs(te + k * st);
        const uint32_t e = s_ref[__ldcs(ty + k * st)];     // Ext of the split model, or the caller's reference
        const uint64_t t1000 = 1000ull * (uint64_t)t;
        for (uint32_t j = 0; j < a.n_alpha; ++j)
            s_viol[j * kQosThreads + tid] += (t1000 > (uint64_t)s_alpha[j] * e) ? 1u : 0u;
        const double rr = __ddiv_rn(__ll2double_rn(t), __uint2double_rn(e));
        rs = __dadd_rn(rs, rr);
        rq = __dadd_rn(rq, __dmul_rn(rr, rr));
    }
    for (uint32_t j = 0; j < a.n_alpha; ++j) a.viol[r * a.n_alpha + j] = s_viol[j * kQosThreads + tid];
    a.rr[2 * r] = rs;
    a.rr[2 * r + 1] = rq;
}

size_t qos_smem_bytes(const QosArgs& a, uint32_t qcap)
{
    return 4 * ((size_t)2 * a.n_types + 1 + a.n_alpha + a.n_blocks_total) + 4 * (size_t)3 * qcap * kQosThreads +
           4 * (size_t)a.n_alpha * kQosThreads + 8 * (size_t)a.n_types + 16;
}

// qcap: kQosQueue (the fast form: many CTAs per SM) or kQosQueueBig (the host's re-run after an overflow)
cudaError_t launch_qos(const QosArgs& a, cudaStream_t st, uint32_t qcap)
{
    if (a.n_rep == 0) return cudaSuccess;
    const size_t sm = qos_smem_bytes(a, qcap);
    const bool big = qcap > kQosQueue;
    const auto kern = (a.policy == 2u) ? (big ? qos_kernel<true, kQosQueueBig> : qos_kernel<true, kQosQueue>)
                                       : (big ? qos_kernel<false, kQosQueueBig> : qos_kernel<false, kQosQueue>);
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    const uint32_t grid = (uint32_t)((a.n_rep + kQosThreads - 1) / kQosThreads);
    kern<<<grid, kQosThreads, sm, st>>>(a);
    return cudaGetLastError();
}

}  // namespace splitga
