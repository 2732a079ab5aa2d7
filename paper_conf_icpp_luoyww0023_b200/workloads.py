"""Seeded synthetic inputs shared by the tests, bench.py and the oracle legs.

This module holds NONE of the method's arithmetic (no fitness, no Philox, no
GA operator): it only draws operator-latency chains, cut-overhead profiles and
candidate bitset populations with numpy's PCG64, so the same inputs can be fed
to the CUDA path and to the CPU oracle.  The recipe is DESIGN.md §4.

Chain shapes follow the paper's workloads: per-operator latencies profiled in
integer ns (P@18308-18385), Table 1's models (P@29872-30320: YOLOv2 84 ops /
10.8 ms, GoogLeNet 142 / 13.2, ResNet50 122 / 28.35, VGG19 44 / 67.5, GPT-2
2534 / 20.4) and BASELINE.json's configs (ResNet-50 ~175 ops, VGG-16,
MobileNetV2, BERT-base ~400 ops, a 1024-op synthetic chain).  Early operators
are longer and cutting early costs more overhead (§2.4 observations,
P@12726-14633): latency weights and cut overheads both decay with the stage.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

# role -> relative latency weight
_ROLE_W = {
    "conv": 1.0, "bn": 0.15, "relu": 0.08, "add": 0.10, "pool": 0.12, "fc": 0.6,
    "dw": 0.35, "pw": 0.7, "matmul": 1.0, "softmax": 0.25, "ln": 0.12, "gelu": 0.15,
    "op": 1.0,
}
_PATTERNS = {
    "resnet": ["conv", "bn", "relu", "conv", "bn", "relu", "conv", "bn", "add", "relu"],
    "vgg": ["conv", "relu", "conv", "relu", "pool"],
    "mobilenet": ["pw", "bn", "relu", "dw", "bn", "relu", "pw", "bn", "add"],
    "bert": ["matmul", "matmul", "matmul", "matmul", "softmax", "matmul", "add", "ln",
             "matmul", "gelu", "matmul", "add", "ln"],
    "yolo": ["conv", "bn", "relu", "pool"],
    "inception": ["conv", "relu", "conv", "relu", "pool", "conv", "relu", "add"],
    "gpt": ["ln", "matmul", "softmax", "matmul", "add", "ln", "matmul", "gelu", "matmul", "add"],
    "synthetic": ["op"],
}
_STAGE_F = (1.0, 0.72, 0.52, 0.38)   # later stages: smaller tensors, shorter ops


@dataclass(frozen=True)
class ChainSpec:
    name: str
    n_ops: int
    total_ns: int
    pattern: str
    seed: int


# model presets: BASELINE.json configs and PAPER.md Table 1
CHAINS = {
    "resnet50_175": ChainSpec("resnet50_175", 175, 28_350_000, "resnet", 1750),
    "resnet50_122": ChainSpec("resnet50_122", 122, 28_350_000, "resnet", 1220),
    "vgg16": ChainSpec("vgg16", 37, 60_000_000, "vgg", 370),
    "mobilenetv2": ChainSpec("mobilenetv2", 105, 10_000_000, "mobilenet", 1050),
    "bert_base": ChainSpec("bert_base", 400, 20_000_000, "bert", 4000),
    "synthetic_1024": ChainSpec("synthetic_1024", 1024, 1 << 24, "synthetic", 10240),
    "yolov2": ChainSpec("yolov2", 84, 10_800_000, "yolo", 840),
    "googlenet": ChainSpec("googlenet", 142, 13_200_000, "inception", 1420),
    "vgg19": ChainSpec("vgg19", 44, 67_500_000, "vgg", 440),
    "gpt2": ChainSpec("gpt2", 2534, 20_400_000, "gpt", 25340),
}


def _stage(i: np.ndarray, n: int) -> np.ndarray:
    return np.minimum((4 * i) // n, 3)


def chain_latencies(spec: ChainSpec) -> np.ndarray:
    """int64 ns latencies, sum close to spec.total_ns, every op >= 1 ns."""
    rng = np.random.Generator(np.random.PCG64(spec.seed))
    n = spec.n_ops
    i = np.arange(n)
    pat = _PATTERNS[spec.pattern]
    role = np.array([_ROLE_W[pat[j % len(pat)]] for j in range(n)])
    stage_f = np.array(_STAGE_F)[_stage(i, n)]
    jitter = rng.uniform(0.75, 1.25, size=n)
    w = role * stage_f * jitter
    lat = np.floor(spec.total_ns * w / w.sum()).astype(np.int64)
    return np.maximum(lat, 1)


def overhead_profile(spec: ChainSpec, lat: np.ndarray, rho_min: float = 0.02, rho_max: float = 0.15) -> np.ndarray:
    """int64 ns overhead of a cut after op p (p in [0, n-2]); larger for early cuts."""
    rng = np.random.Generator(np.random.PCG64(spec.seed + 1))
    n = spec.n_ops
    T = int(lat.sum())
    p = np.arange(n - 1)
    act = np.power(0.5, _stage(p + 1, n).astype(np.float64)) * rng.uniform(0.75, 1.25, size=n - 1)
    a = act / act.max()
    return np.floor(T * (rho_min + (rho_max - rho_min) * a)).astype(np.int64)


def constant_overhead(lat: np.ndarray, frac: float = 0.05) -> tuple[np.ndarray, int]:
    """Constant per-cut overhead delta = floor(frac * T) (the DP configs)."""
    T = int(lat.sum())
    delta = int(np.floor(frac * T))
    return np.full(len(lat) - 1, delta, dtype=np.int64), delta


def chain(name: str, overhead: str = "profile"):
    """(latencies, overheads) for a preset; overhead in {'profile','const','zero'}."""
    spec = CHAINS[name]
    lat = chain_latencies(spec)
    if overhead == "profile":
        ovh = overhead_profile(spec, lat)
    elif overhead == "const":
        ovh, _ = constant_overhead(lat)
    elif overhead == "zero":
        ovh = np.zeros(spec.n_ops - 1, dtype=np.int64)
    else:
        raise ValueError(overhead)
    return lat, ovh


def c1_chain(seed: int = 12, overhead: str = "profile"):
    """C1: a 12-operator chain, latencies uniform in [1, 1000] us (integer ns)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    lat = rng.integers(1_000, 1_000_001, size=12, dtype=np.int64)
    if overhead == "profile":
        T = int(lat.sum())
        ovh = np.floor(T * np.linspace(0.15, 0.02, 11) * rng.uniform(0.8, 1.2, size=11)).astype(np.int64)
    elif overhead == "const":
        ovh = np.full(11, int(0.05 * lat.sum()), dtype=np.int64)
    elif overhead == "zero":
        ovh = np.zeros(11, dtype=np.int64)
    elif overhead == "ties":   # a tie-rich chain: every op 1000 ns, no overhead
        lat = np.full(12, 1000, dtype=np.int64)
        ovh = np.zeros(11, dtype=np.int64)
    else:
        raise ValueError(overhead)
    return lat, ovh


def random_chain(n: int, seed: int, lo: int = 1, hi: int = 1_000_000, ovh_hi: int = 0):
    rng = np.random.Generator(np.random.PCG64(seed))
    lat = rng.integers(lo, hi + 1, size=n, dtype=np.int64)
    ovh = rng.integers(0, ovh_hi + 1, size=n - 1, dtype=np.int64) if ovh_hi > 0 else np.zeros(n - 1, np.int64)
    return lat, ovh


def words(n_ops: int) -> int:
    return (n_ops - 1 + 63) // 64


def pack_positions(rows_positions, n_ops: int) -> np.ndarray:
    """Pack lists of cut positions into the [N][W] u64 bitset layout (bit p of word p>>6)."""
    W = words(n_ops)
    out = np.zeros((len(rows_positions), W), dtype=np.uint64)
    for r, pos in enumerate(rows_positions):
        for p in pos:
            out[r, p >> 6] |= np.uint64(1) << np.uint64(p & 63)
    return out


def sparse_population(n_ops: int, n_cand: int, seed: int, k_lo: int = 2, k_hi: int = 32) -> np.ndarray:
    """Bitsets with k ~ U[k_lo, k_hi] blocks, cut positions uniform without replacement."""
    rng = np.random.Generator(np.random.PCG64(seed))
    W = words(n_ops)
    m = n_ops - 1
    k_hi = min(k_hi, n_ops)
    out = np.zeros((n_cand, W), dtype=np.uint64)
    ks = rng.integers(k_lo, k_hi + 1, size=n_cand)
    # vectorised: random keys per position, take the (k-1) smallest
    chunk = 1 << 16
    for s in range(0, n_cand, chunk):
        e = min(n_cand, s + chunk)
        keys = rng.random((e - s, m))
        order = np.argsort(keys, axis=1)
        ranks = np.empty_like(order)
        np.put_along_axis(ranks, order, np.arange(m)[None, :].repeat(e - s, 0), axis=1)
        sel = ranks < (ks[s:e, None] - 1)
        for w in range(W):
            blk = sel[:, w * 64:(w + 1) * 64]
            weights = (np.uint64(1) << np.arange(blk.shape[1], dtype=np.uint64))
            out[s:e, w] = (blk.astype(np.uint64) * weights[None, :]).sum(axis=1, dtype=np.uint64)
    return out


def dense_population(n_ops: int, n_cand: int, seed: int, with_padding: bool = False) -> np.ndarray:
    """Bernoulli(1/2) bitsets (the C5 dense variant); optionally random padding bits."""
    rng = np.random.Generator(np.random.PCG64(seed))
    W = words(n_ops)
    out = rng.integers(0, np.iinfo(np.uint64).max, size=(n_cand, W), dtype=np.uint64, endpoint=True)
    if not with_padding:
        pad = (n_ops - 1) & 63
        if pad:
            out[:, W - 1] &= np.uint64((1 << pad) - 1)
    return out


def uniform_k_population_fast(n_ops: int, n_cand: int, seed: int, k_lo: int = 2, k_hi: int = 32) -> np.ndarray:
    """Large-N sparse population (C5) without the O(N*n) sort: draw k-1 positions
    with replacement-and-retry per row via numpy vector ops (duplicates collapse,
    so k is <= the drawn value)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    W = words(n_ops)
    m = n_ops - 1
    ks = rng.integers(k_lo, min(k_hi, n_ops) + 1, size=n_cand)
    kmax = int(ks.max()) - 1 if n_cand else 0
    out = np.zeros((n_cand, W), dtype=np.uint64)
    if kmax <= 0:
        return out
    pos = rng.integers(0, m, size=(n_cand, kmax))
    valid = np.arange(kmax)[None, :] < (ks[:, None] - 1)
    rows = np.repeat(np.arange(n_cand), kmax)[valid.reshape(-1)]
    p = pos.reshape(-1)[valid.reshape(-1)]
    bit = np.left_shift(np.uint64(1), (p & 63).astype(np.uint64))
    np.bitwise_or.at(out, (rows, p >> 6), bit)
    return out


def qos_requests(n_rep: int, n_req: int, lam_ns: int, n_types: int, seed: int):
    """Poisson request streams for the f2 simulator (§5.1, Table 2 P@31725-32980:
    mean arrival interval lambda, here in ns): per replica, exponential
    inter-arrival gaps rounded to integer ns (cumulative, starting at the first
    gap) and a model type uniform in [0, n_types).  Returns (arrival int64
    [n_rep, n_req], type int32 [n_rep, n_req]), replica-major; the simulator
    takes the request-major transposes (np.ascontiguousarray(x.T))."""
    rng = np.random.default_rng(seed)
    gaps = np.rint(rng.exponential(float(lam_ns), size=(n_rep, n_req))).astype(np.int64)
    arrival = np.cumsum(gaps, axis=1)
    types = rng.integers(0, n_types, size=(n_rep, n_req), dtype=np.int32)
    return arrival, types


def random_blocks(n_types: int, seed: int, k_lo: int = 1, k_hi: int = 6, lo: int = 200_000, hi: int = 20_000_000):
    """Random per-model block lists (ns) for simulator tests: k in [k_lo, k_hi]
    blocks per model, each uniform in [lo, hi)."""
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(n_types):
        k = int(rng.integers(k_lo, k_hi + 1))
        out.append([int(x) for x in rng.integers(lo, hi, size=k)])
    return out
