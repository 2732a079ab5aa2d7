"""ctypes binding of include/split_ga.h — argument marshalling only.

Every step of the GA split search runs in libsplit_ga.so (sm_100a kernels +
the C++ host runtime).  There is no Python or CPU fallback: if the library is
missing or fails to load, importing this module raises.  torch is used only
for device memory (tensor data pointers) and streams; the ABI itself takes
plain pointers and sizes.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SPLIT_LIB") or os.path.join(_PKG, "lib", "libsplit_ga.so")   # SPLIT_LIB: tuning A/B only

SPLIT_OK = 0
SPLIT_E_INVAL, SPLIT_E_RANGE, SPLIT_E_ALIGN, SPLIT_E_NOMEM, SPLIT_E_CUDA, SPLIT_E_NCCL, SPLIT_E_STATE = range(-1, -8, -1)


class split_ga_params(C.Structure):
    _fields_ = [
        ("pop_size", C.c_uint32), ("n_elite", C.c_uint32), ("tournament_size", C.c_uint32),
        ("p_crossover", C.c_double), ("p_mutation", C.c_double),
        ("k_min", C.c_uint32), ("k_max", C.c_uint32), ("front_skip", C.c_uint32),
        ("stall_generations", C.c_uint32), ("cut_overhead_ns", C.POINTER(C.c_int64)),
        ("island_id", C.c_uint32), ("n_islands", C.c_uint32), ("islands_per_device", C.c_uint32),
        ("migration_interval", C.c_uint32), ("n_migrants", C.c_uint32),
        ("comm", C.c_void_p), ("device", C.c_int), ("stream", C.c_void_p),
    ]


class split_best_t(C.Structure):
    _fields_ = [
        ("bits", C.POINTER(C.c_uint64)), ("fitness", C.c_double), ("k", C.c_uint32),
        ("var_num", C.c_int64), ("s1", C.c_uint64), ("s2", C.c_uint64), ("overhead_ns", C.c_uint64),
        ("expected_wait_ns", C.c_double), ("generation_found", C.c_uint32),
        ("generations_run", C.c_uint32), ("evaluations", C.c_uint64),
    ]


class split_request(C.Structure):
    _fields_ = [("type_id", C.c_uint32), ("arrival_ns", C.c_int64), ("ext_ns", C.c_int64), ("ext_left_ns", C.c_int64)]


class split_queue_state(C.Structure):
    _fields_ = [("now_ns", C.c_int64), ("alpha", C.c_double), ("n", C.c_uint32),
                ("queue", C.POINTER(split_request)), ("incoming", split_request)]


class split_k_result(C.Structure):
    _fields_ = [("k", C.c_uint32), ("fitness", C.c_double), ("expected_wait_ns", C.c_double),
                ("overhead_ns", C.c_uint64), ("var_num", C.c_int64), ("s1", C.c_uint64), ("s2", C.c_uint64),
                ("cost_ns", C.c_double)]


class split_run_stats(C.Structure):
    _fields_ = [("launches", C.c_uint64), ("ms_total", C.c_float), ("ms_loop", C.c_float),
                ("general_selects", C.c_uint32), ("fast_selects", C.c_uint32)]


class SplitError(RuntimeError):
    def __init__(self, code: int, where: str, detail: str):
        super().__init__(f"{where}: {code} {detail}")
        self.code = code


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_icpp_luoyww0023_b200.build` "
                          "(the CUDA library is the only implementation; there is no fallback)")
    L = C.CDLL(LIB_PATH)
    P = C.POINTER
    sig = {
        "split_ga_params_default": (None, [P(split_ga_params)]),
        "split_ga_create": (C.c_int, [P(C.c_int64), C.c_uint32, P(split_ga_params), P(C.c_void_p)]),
        "split_words": (C.c_uint32, [C.c_void_p]),
        "split_eval_batch": (C.c_int, [C.c_void_p, C.c_void_p, C.c_uint64, C.c_void_p]),
        "split_eval_batch_host": (C.c_int, [C.c_void_p, C.c_void_p, C.c_uint64, C.c_void_p]),
        "split_ga_run": (C.c_int, [C.c_void_p, C.c_uint32, C.c_uint64, P(split_best_t)]),
        "split_ga_set_chain": (C.c_int, [C.c_void_p, P(C.c_int64), P(C.c_int64)]),
        "split_k_sweep": (C.c_int, [C.c_void_p, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint64, P(split_k_result),
                                    P(C.c_uint32)]),
        "split_ga_population": (C.c_int, [C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p]),
        "split_preempt_decide": (C.c_int, [P(split_queue_state), P(C.c_uint32)]),
        "split_qos_simulate": (C.c_int, [P(C.c_int64), P(C.c_uint32), C.c_uint32, C.c_uint32, P(C.c_uint32),
                                         C.c_uint32, C.c_uint64, C.c_uint32, C.c_void_p, C.c_void_p, C.c_void_p,
                                         C.c_void_p, C.c_void_p, C.c_int, C.c_void_p]),
        "split_qos_simulate_elastic": (C.c_int, [P(C.c_int64), P(C.c_uint32), P(C.c_int64), P(C.c_int64), C.c_uint32, C.c_uint32,
                                                 C.c_uint32, P(C.c_uint32), C.c_uint32, C.c_uint64, C.c_uint32,
                                                 C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_int,
                                                 C.c_void_p]),
        "split_comm_unique_id": (C.c_int, [C.c_void_p]),
        "split_comm_init": (C.c_int, [C.c_void_p, C.c_int, C.c_int, C.c_int, P(C.c_void_p)]),
        "split_comm_destroy": (None, [C.c_void_p]),
        "split_ga_destroy": (None, [C.c_void_p]),
        "split_strerror": (C.c_char_p, [C.c_int]),
        "split_last_error": (C.c_char_p, []),
        "split_selftest_philox": (C.c_int, [C.c_int, C.c_void_p, C.c_uint32, C.c_void_p]),
        "split_selftest_dexp": (C.c_int, [C.c_int, C.c_void_p, C.c_uint32, C.c_void_p]),
        "split_last_run_stats": (C.c_int, [C.c_void_p, P(split_run_stats)]),
        "split_exhaustive": (C.c_int, [C.c_void_p, P(split_best_t), C.c_void_p, C.c_void_p]),
        "split_dp_min_s2": (C.c_int, [C.c_void_p, C.c_uint32, C.c_void_p]),
        "split_heatmap2": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]),
        "split_block_times": (C.c_int, [C.c_void_p, C.c_void_p, C.c_uint32, C.c_void_p, C.c_void_p, C.c_uint32,
                                        P(C.c_uint32)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    return L


_lib = _load()
EXPORTED = ("split_ga_params_default", "split_ga_create", "split_words", "split_eval_batch",
            "split_eval_batch_host", "split_ga_run", "split_ga_population", "split_preempt_decide",
            "split_comm_unique_id", "split_comm_init", "split_comm_destroy", "split_ga_destroy",
            "split_strerror", "split_last_error", "split_selftest_philox", "split_selftest_dexp",
            "split_last_run_stats", "split_exhaustive", "split_dp_min_s2", "split_qos_simulate", "split_ga_set_chain", "split_k_sweep",
            "split_qos_simulate_elastic", "split_block_times", "split_heatmap2")


def lib():
    return _lib


def _check(rc: int, where: str):
    if rc != SPLIT_OK:
        raise SplitError(rc, where, f"{_lib.split_strerror(rc).decode()}: {_lib.split_last_error().decode()}")


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def words(n_ops: int) -> int:
    return (n_ops - 1 + 63) // 64


# ---------------------------------------------------------------- same names as the C ABI
def split_ga_params_default() -> dict:
    p = split_ga_params()
    _lib.split_ga_params_default(C.byref(p))
    return {f: getattr(p, f) for f, _ in split_ga_params._fields_ if f not in ("cut_overhead_ns", "comm", "stream")}


def split_preempt_decide(now_ns: int, alpha: float, queue, incoming) -> int:
    """queue: list of (type_id, arrival_ns, ext_ns, ext_left_ns), head first; incoming likewise."""
    n = len(queue)
    arr = (split_request * max(n, 1))()
    for i, r in enumerate(queue):
        arr[i] = split_request(*[int(x) for x in r])
    q = split_queue_state(int(now_ns), float(alpha), n, arr if n else None, split_request(*[int(x) for x in incoming]))
    pos = C.c_uint32(0)
    _check(_lib.split_preempt_decide(C.byref(q), C.byref(pos)), "split_preempt_decide")
    return int(pos.value)


def split_qos_simulate(blocks, arrival, type_id, alpha_milli, policy: int = 1, *, device: int | None = None,
                       stream=None, unsplit=None, d_max: int = 0, s_max: int = 0, ref=None):
    """f2 QoS simulator (include/split_ga.h).  blocks: per model type, its block
    times (ns); arrival: device int64 tensor [n_req, n_rep] (request-major);
    type_id: device int32 tensor of the same shape.  Returns device tensors
    (t_ete [n_req, n_rep] int64, violations [n_rep, n_alpha] int32 (uint32 bits),
    rr [n_rep, 2] f64).  policy 2 = f4 elastic splitting
    (split_qos_simulate_elastic): unsplit = per-type unsplit latency (ns),
    d_max / s_max = the density and same-type thresholds (R23); ref = per-type
    latency reference for violations and RR (None = the split Ext).
    device defaults to arrival's device, stream to that device's current torch
    stream (the one the output tensors are allocated on)."""
    import torch
    n_req, n_rep = arrival.shape
    if device is None:
        device = arrival.device.index if arrival.device.index is not None else torch.cuda.current_device()
    if stream is None:
        stream = torch.cuda.current_stream(device)
    flat = np.ascontiguousarray(np.concatenate([np.asarray(b, dtype=np.int64) for b in blocks]))
    nb = np.ascontiguousarray(np.array([len(b) for b in blocks], dtype=np.uint32))
    al = np.ascontiguousarray(np.asarray(alpha_milli, dtype=np.uint32))
    dev = arrival.device
    t_ete = torch.empty((n_req, n_rep), dtype=torch.int64, device=dev)
    viol = torch.empty((n_rep, max(len(al), 1)), dtype=torch.int32, device=dev)
    rr = torch.empty((n_rep, 2), dtype=torch.float64, device=dev)
    assert arrival.dtype == torch.int64 and arrival.is_contiguous()
    assert type_id.dtype == torch.int32 and type_id.is_contiguous() and type_id.shape == arrival.shape
    if policy == 2:
        un = np.ascontiguousarray(np.asarray(unsplit, dtype=np.int64))
        assert un.shape == (len(blocks),)
        rf = None if ref is None else np.ascontiguousarray(np.asarray(ref, dtype=np.int64))
        if rf is not None and rf.shape != (len(blocks),):
            raise ValueError("ref needs one entry per model type")
        _check(lib().split_qos_simulate_elastic(flat.ctypes.data_as(C.POINTER(C.c_int64)),
                                                nb.ctypes.data_as(C.POINTER(C.c_uint32)),
                                                un.ctypes.data_as(C.POINTER(C.c_int64)),
                                                None if rf is None else rf.ctypes.data_as(C.POINTER(C.c_int64)),
                                                len(blocks), d_max, s_max,
                                                al.ctypes.data_as(C.POINTER(C.c_uint32)), len(al), n_rep, n_req,
                                                arrival.data_ptr(), type_id.data_ptr(), t_ete.data_ptr(),
                                                viol.data_ptr(), rr.data_ptr(), device, _stream_handle(stream)),
               "split_qos_simulate_elastic")
        return t_ete, viol, rr
    _check(lib().split_qos_simulate(flat.ctypes.data_as(C.POINTER(C.c_int64)), nb.ctypes.data_as(C.POINTER(C.c_uint32)),
                                    len(blocks), policy, al.ctypes.data_as(C.POINTER(C.c_uint32)), len(al), n_rep,
                                    n_req, arrival.data_ptr(), type_id.data_ptr(), t_ete.data_ptr(), viol.data_ptr(),
                                    rr.data_ptr(), device, _stream_handle(stream)), "split_qos_simulate")
    return t_ete, viol, rr


def split_block_times(latencies_ns, cut_overhead_ns, bits) -> list[int]:
    """Block execution times (ns) of one split (include/split_ga.h split_block_times)."""
    lat = np.ascontiguousarray(latencies_ns, dtype=np.int64)
    ovh = None if cut_overhead_ns is None else np.ascontiguousarray(cut_overhead_ns, dtype=np.int64)
    b = np.ascontiguousarray(bits, dtype=np.uint64)
    if ovh is not None and ovh.size != lat.size - 1:
        raise ValueError("cut_overhead_ns needs n_ops - 1 entries")
    if b.size < words(lat.size):
        raise ValueError("bits needs ceil((n_ops-1)/64) words")
    out = np.zeros(lat.size, dtype=np.int64)           # at most n_ops blocks
    k = C.c_uint32(0)
    _check(_lib.split_block_times(_ptr(lat), None if ovh is None else _ptr(ovh), lat.size, _ptr(b), _ptr(out),
                                  out.size, C.byref(k)), "split_block_times")
    return [int(x) for x in out[:k.value]]


def split_comm_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(_lib.split_comm_unique_id(buf), "split_comm_unique_id")
    return bytes(buf)


def split_comm_init(uid: bytes, rank: int, world: int, device: int) -> int:
    buf = (C.c_uint8 * 128).from_buffer_copy(uid)
    h = C.c_void_p()
    _check(_lib.split_comm_init(buf, rank, world, device, C.byref(h)), "split_comm_init")
    return h.value


def split_comm_destroy(comm) -> None:
    if comm:
        _lib.split_comm_destroy(C.c_void_p(comm))


def split_selftest_philox(ctr_key: np.ndarray, device: int = 0) -> np.ndarray:
    ck = np.ascontiguousarray(ctr_key, dtype=np.uint32).reshape(-1, 6)
    out = np.zeros((ck.shape[0], 4), dtype=np.uint32)
    _check(_lib.split_selftest_philox(device, _ptr(ck), ck.shape[0], _ptr(out)), "split_selftest_philox")
    return out


def split_selftest_dexp(z: np.ndarray, device: int = 0) -> np.ndarray:
    z = np.ascontiguousarray(z, dtype=np.float64)
    out = np.zeros_like(z)
    _check(_lib.split_selftest_dexp(device, _ptr(z), z.size, _ptr(out)), "split_selftest_dexp")
    return out


class SplitGA:
    """One split_ga_t handle (split_ga_create ... split_ga_destroy)."""

    def __init__(self, latencies_ns, cut_overhead_ns=None, *, device: int = 0, stream=None, comm=None, **params):
        lat = np.ascontiguousarray(latencies_ns, dtype=np.int64)
        self.n_ops = int(lat.size)
        p = split_ga_params()
        _lib.split_ga_params_default(C.byref(p))
        for k, v in params.items():
            if not hasattr(p, k):
                raise TypeError(f"unknown GA parameter {k}")
            setattr(p, k, v)
        self._ovh = None
        if cut_overhead_ns is not None:
            self._ovh = np.ascontiguousarray(cut_overhead_ns, dtype=np.int64)
            if self._ovh.size != self.n_ops - 1:
                raise ValueError("cut_overhead_ns needs n_ops - 1 entries")
            p.cut_overhead_ns = self._ovh.ctypes.data_as(C.POINTER(C.c_int64))
        p.device = device
        if stream is None:
            stream = _current_stream(device)
        p.stream = C.c_void_p(_stream_handle(stream))
        p.comm = C.c_void_p(comm) if comm else None
        self.params = p
        h = C.c_void_p()
        _check(_lib.split_ga_create(lat.ctypes.data_as(C.POINTER(C.c_int64)), self.n_ops, C.byref(p), C.byref(h)),
               "split_ga_create")
        self._h = h
        self.W = int(_lib.split_words(h))

    # a2 on device buffers (torch tensors or raw pointers)
    def eval_batch(self, bits, n_cand: int | None = None, out=None):
        bptr, n = _dev_ptr(bits), n_cand
        if n is None:
            n = int(bits.shape[0])
        if out is None:
            import torch
            out = torch.empty(n, dtype=torch.float64, device=bits.device)
        _check(_lib.split_eval_batch(self._h, C.c_void_p(bptr), n, C.c_void_p(_dev_ptr(out))), "split_eval_batch")
        return out

    # a2 through host buffers (copies inside the call)
    def eval_batch_host(self, bits: np.ndarray, out: np.ndarray | None = None) -> np.ndarray:
        b = np.ascontiguousarray(bits, dtype=np.uint64)
        n = b.shape[0] if b.ndim == 2 else b.size // max(self.W, 1)
        if out is None:
            out = np.empty(n, dtype=np.float64)
        _check(_lib.split_eval_batch_host(self._h, _ptr(b), n, _ptr(out)), "split_eval_batch_host")
        return out

    def k_sweep(self, k_lo: int, k_hi: int, generations: int, seed: int):
        """f3: fixed-k GA per k in [k_lo, k_hi]; returns (k_best, [per-k dicts])."""
        res = (split_k_result * (k_hi - k_lo + 1))()
        kb = C.c_uint32(0)
        _check(_lib.split_k_sweep(self._h, k_lo, k_hi, generations, seed, res, C.byref(kb)), "split_k_sweep")
        return kb.value, [{f: getattr(r, f) for f, _ in split_k_result._fields_} for r in res]

    def set_chain(self, latencies_ns, cut_overhead_ns=None) -> None:
        """Replace the handle's chain (same n_ops): host arrays, uploaded on the handle's stream."""
        lat = np.ascontiguousarray(latencies_ns, dtype=np.int64)
        ovh = None if cut_overhead_ns is None else np.ascontiguousarray(cut_overhead_ns, dtype=np.int64)
        if lat.size != self.n_ops:
            raise ValueError(f"latencies_ns needs n_ops = {self.n_ops} entries (got {lat.size})")
        if ovh is not None and ovh.size != self.n_ops - 1:
            raise ValueError(f"cut_overhead_ns needs n_ops - 1 = {self.n_ops - 1} entries (got {ovh.size})")
        self._keep_chain = (lat, ovh)          # the copy is staged before the call returns; kept for clarity
        _check(_lib.split_ga_set_chain(self._h, lat.ctypes.data_as(C.POINTER(C.c_int64)),
                                       None if ovh is None else ovh.ctypes.data_as(C.POINTER(C.c_int64))),
               "split_ga_set_chain")

    def run(self, generations: int, seed: int) -> dict:
        bits = np.zeros(max(self.W, 1), dtype=np.uint64)
        best = split_best_t()
        best.bits = bits.ctypes.data_as(C.POINTER(C.c_uint64))
        _check(_lib.split_ga_run(self._h, generations, seed, C.byref(best)), "split_ga_run")
        out = {f: getattr(best, f) for f, _ in split_best_t._fields_ if f != "bits"}
        out["bits"] = bits
        return out

    # f1: exact optimum over all 2^(n_ops-1) splits (and optionally min V / argmin per k)
    def exhaustive(self, per_k: bool = False) -> dict:
        bits = np.zeros(max(self.W, 1), dtype=np.uint64)
        best = split_best_t()
        best.bits = bits.ctypes.data_as(C.POINTER(C.c_uint64))
        kmax = int(self.params.k_max)
        mv = np.zeros(kmax + 1, dtype=np.int64) if per_k else None
        am = np.zeros(kmax + 1, dtype=np.uint64) if per_k else None
        _check(_lib.split_exhaustive(self._h, C.byref(best), _ptr(mv) if per_k else None,
                                     _ptr(am) if per_k else None), "split_exhaustive")
        out = {f: getattr(best, f) for f, _ in split_best_t._fields_ if f != "bits"}
        out["bits"] = bits
        if per_k:
            out["min_v_per_k"] = mv
            out["argmin_per_k"] = am
        return out

    # f1: the two-cut map (Fig. 2 analog) into device tensors
    def heatmap2(self, var_out=None, ov_out=None, fit_out=None):
        """Returns (V int64, OV int64 (uint64 bits), fitness f64) device tensors of shape
        [n_ops-1, n_ops-1], entry [a][b] for a <= b; pass tensors to reuse buffers."""
        import torch
        m = self.n_ops - 1
        dev = torch.device("cuda", self.params.device)
        var_out = torch.empty((m, m), dtype=torch.int64, device=dev) if var_out is None else var_out
        ov_out = torch.empty((m, m), dtype=torch.int64, device=dev) if ov_out is None else ov_out
        fit_out = torch.empty((m, m), dtype=torch.float64, device=dev) if fit_out is None else fit_out
        for t in (var_out, ov_out, fit_out):
            if t.numel() < m * m or not t.is_contiguous():
                raise ValueError("heatmap2 outputs need (n_ops-1)^2 contiguous entries")
        _check(_lib.split_heatmap2(self._h, C.c_void_p(_dev_ptr(var_out)), C.c_void_p(_dev_ptr(ov_out)),
                                   C.c_void_p(_dev_ptr(fit_out))), "split_heatmap2")
        return var_out, ov_out, fit_out

    # f1: min S2 per block count by the O(k n^2) DP
    def dp_min_s2(self, k_max: int) -> np.ndarray:
        out = np.zeros(k_max + 1, dtype=np.uint64)
        _check(_lib.split_dp_min_s2(self._h, k_max, _ptr(out)), "split_dp_min_s2")
        return out

    def population(self, island: int = 0):
        N = self.params.pop_size
        bits = np.zeros((N, self.W), dtype=np.uint64)
        fit = np.zeros(N, dtype=np.float64)
        _check(_lib.split_ga_population(self._h, island, _ptr(bits), _ptr(fit)), "split_ga_population")
        return bits, fit

    def last_run_stats(self) -> dict:
        s = split_run_stats()
        _check(_lib.split_last_run_stats(self._h, C.byref(s)), "split_last_run_stats")
        return {f: getattr(s, f) for f, _ in split_run_stats._fields_}

    def close(self):
        if getattr(self, "_h", None):
            _lib.split_ga_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


def _current_stream(device: int):
    """torch's current stream on `device` (where torch allocates the caller's
    tensors); 0 (legacy default stream) when torch has no usable CUDA."""
    try:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream(device)
    except Exception:
        pass
    return 0


def _stream_handle(stream) -> int:
    if stream is None:
        return 0
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


def _dev_ptr(x) -> int:
    if isinstance(x, int):
        return x
    return int(x.data_ptr())
