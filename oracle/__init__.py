"""CPU oracle for the SPLIT GA split search — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
and ``--impl reference`` legs may import this package.  The product
(``paper_conf_icpp_luoyww0023_b200``) never imports it and shares no code,
header, table or constant with it.

``liboracle.so`` is built from ``split_oracle.c`` (plain C99, single thread,
``-O2 -ffp-contract=off -fno-fast-math``).  This module is argument
marshalling only; every number comes from the C code (or, for Algorithm 1,
from ``oracle/preempt.py`` in exact rationals).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "split_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=gnu99", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-Wall"]


def build(force: bool = False) -> str:
    """Compile liboracle.so in-tree (gcc)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "split_oracle.h"))):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class Stats(C.Structure):
    _fields_ = [("fitness", C.c_double), ("k", C.c_uint32), ("var_num", C.c_int64),
                ("s1", C.c_uint64), ("s2", C.c_uint64), ("overhead", C.c_uint64), ("T", C.c_uint64)]


class BruteResult(C.Structure):
    _fields_ = [("fitness", C.c_double), ("bits", C.c_uint64), ("k", C.c_uint32), ("var_num", C.c_int64)]


class GAParams(C.Structure):
    _fields_ = [("pop_size", C.c_uint32), ("n_elite", C.c_uint32), ("tournament_size", C.c_uint32),
                ("p_crossover", C.c_double), ("p_mutation", C.c_double),
                ("k_min", C.c_uint32), ("k_max", C.c_uint32), ("front_skip", C.c_uint32),
                ("stall_generations", C.c_uint32), ("n_islands", C.c_uint32), ("island_base", C.c_uint32),
                ("migration_interval", C.c_uint32), ("n_migrants", C.c_uint32)]


class GABest(C.Structure):
    _fields_ = [("bits", C.POINTER(C.c_uint64)), ("fitness", C.c_double), ("k", C.c_uint32),
                ("var_num", C.c_int64), ("s1", C.c_uint64), ("s2", C.c_uint64), ("overhead", C.c_uint64),
                ("generation_found", C.c_uint32), ("generations_run", C.c_uint32), ("evaluations", C.c_uint64)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        L = _lib
        P64, PU64, PD = C.POINTER(C.c_int64), C.POINTER(C.c_uint64), C.POINTER(C.c_double)
        L.or_philox4x32_10.argtypes = [C.POINTER(C.c_uint32), C.POINTER(C.c_uint32), C.POINTER(C.c_uint32)]
        L.or_dexp.argtypes = [C.c_double]
        L.or_dexp.restype = C.c_double
        L.or_fitness.argtypes = [C.c_uint32, P64, P64, PU64, C.c_uint32, C.c_uint32, C.POINTER(Stats)]
        L.or_fitness_batch.argtypes = [C.c_uint32, P64, P64, PU64, C.c_uint64, C.c_uint32, C.c_uint32, PD]
        L.or_fitness_from.argtypes = [C.c_uint32, C.c_int64, C.c_int64, C.c_int64]
        L.or_fitness_from.restype = C.c_double
        L.or_brute.argtypes = [C.c_uint32, P64, P64, C.c_uint32, C.c_uint32, C.POINTER(BruteResult), P64, PU64]
        L.or_dp.argtypes = [C.c_uint32, P64, C.c_int64, C.c_uint32, P64]
        L.or_count_fixed_k.argtypes = [C.c_uint32, C.c_uint32]
        L.or_count_fixed_k.restype = C.c_uint64
        L.or_ga_run.argtypes = [C.c_uint32, P64, P64, C.POINTER(GAParams), C.c_uint32, C.c_uint64,
                                C.POINTER(GABest), PU64, PD]
        L.or_heatmap2.argtypes = [C.c_uint32, P64, P64, P64, PU64, PD]
        L.or_heatmap2.restype = None
        L.or_ga_migrate.argtypes = [C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, PU64, PD]
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(C.POINTER(ct)) if a is not None else None


def words(n: int) -> int:
    return (n - 1 + 63) // 64


def philox(ctr, key):
    c = (C.c_uint32 * 4)(*ctr)
    k = (C.c_uint32 * 2)(*key)
    o = (C.c_uint32 * 4)()
    lib().or_philox4x32_10(c, k, o)
    return tuple(o)


def dexp(z: float) -> float:
    return lib().or_dexp(float(z))


def _chain(lat, ovh):
    lat = np.ascontiguousarray(lat, dtype=np.int64)
    ovh = None if ovh is None else np.ascontiguousarray(ovh, dtype=np.int64)
    return lat, ovh


def fitness(lat, ovh, bits, k_min=1, k_max=None) -> dict:
    lat, ovh = _chain(lat, ovh)
    n = len(lat)
    k_max = n if k_max is None else k_max
    bits = np.ascontiguousarray(bits, dtype=np.uint64).reshape(-1)
    assert bits.size >= words(n)
    s = Stats()
    lib().or_fitness(n, _p(lat, C.c_int64), _p(ovh, C.c_int64), _p(bits, C.c_uint64), k_min, k_max, C.byref(s))
    return {f: getattr(s, f) for f, _ in Stats._fields_}


def fitness_batch(lat, ovh, bits2d, k_min=1, k_max=None) -> np.ndarray:
    lat, ovh = _chain(lat, ovh)
    n = len(lat)
    k_max = n if k_max is None else k_max
    bits2d = np.ascontiguousarray(bits2d, dtype=np.uint64)
    n_cand = bits2d.shape[0] if bits2d.size else 0
    out = np.empty(n_cand, dtype=np.float64)
    lib().or_fitness_batch(n, _p(lat, C.c_int64), _p(ovh, C.c_int64), _p(bits2d, C.c_uint64), n_cand,
                           k_min, k_max, _p(out, C.c_double))
    return out


def fitness_from(k, V, OV, T) -> float:
    return lib().or_fitness_from(k, V, OV, T)


def brute(lat, ovh, k_min=1, k_max=None):
    lat, ovh = _chain(lat, ovh)
    n = len(lat)
    k_max = n if k_max is None else k_max
    r = BruteResult()
    minv = np.zeros(n + 1, dtype=np.int64)
    argm = np.zeros(n + 1, dtype=np.uint64)
    rc = lib().or_brute(n, _p(lat, C.c_int64), _p(ovh, C.c_int64), k_min, k_max, C.byref(r),
                        _p(minv, C.c_int64), _p(argm, C.c_uint64))
    if rc != 0:
        raise ValueError(f"or_brute rc={rc}")
    return {"fitness": r.fitness, "bits": int(r.bits), "k": r.k, "var_num": r.var_num,
            "minV_per_k": minv, "argminV_per_k": argm}


def dp(lat, delta: int, k_max: int) -> np.ndarray:
    lat = np.ascontiguousarray(lat, dtype=np.int64)
    out = np.zeros(k_max + 1, dtype=np.int64)
    rc = lib().or_dp(len(lat), _p(lat, C.c_int64), int(delta), k_max, _p(out, C.c_int64))
    if rc != 0:
        raise ValueError(f"or_dp rc={rc}")
    return out


def count_fixed_k(n: int, k: int) -> int:
    return int(lib().or_count_fixed_k(n, k))


def ga_run(lat, ovh, generations: int, seed: int, *, pop_size, n_elite, tournament_size=4,
           p_crossover=0.9, p_mutation=0.2, k_min=2, k_max=None, front_skip=0, stall_generations=0,
           n_islands=1, migration_interval=0, n_migrants=0, want_population=False):
    lat, ovh = _chain(lat, ovh)
    n = len(lat)
    W = words(n)
    k_max = min(n, 32) if k_max is None else k_max
    prm = GAParams(pop_size, n_elite, tournament_size, p_crossover, p_mutation, k_min, k_max, front_skip,
                   stall_generations, n_islands, 0, migration_interval, n_migrants)
    bits = np.zeros(W, dtype=np.uint64)
    best = GABest()
    best.bits = _p(bits, C.c_uint64)
    pop = np.zeros((n_islands, pop_size, W), dtype=np.uint64) if want_population else None
    fit = np.zeros((n_islands, pop_size), dtype=np.float64) if want_population else None
    rc = lib().or_ga_run(n, _p(lat, C.c_int64), _p(ovh, C.c_int64), C.byref(prm), generations, seed,
                         C.byref(best), _p(pop, C.c_uint64), _p(fit, C.c_double))
    if rc != 0:
        raise ValueError(f"or_ga_run rc={rc}")
    out = {f: getattr(best, f) for f, _ in GABest._fields_ if f != "bits"}
    out["bits"] = bits
    if want_population:
        out["population"] = pop
        out["fitness_all"] = fit
    return out


def heatmap2(lat, ovh):
    """Two-cut map (Fig. 2 analog): (V, OV, fitness), each [n-1][n-1], entry [a][b] for a <= b."""
    lat, ovh = _chain(lat, ovh)
    m = len(lat) - 1
    V = np.zeros((m, m), dtype=np.int64)
    OV = np.zeros((m, m), dtype=np.uint64)
    F = np.zeros((m, m), dtype=np.float64)
    lib().or_heatmap2(len(lat), _p(lat, C.c_int64), _p(ovh, C.c_int64), _p(V, C.c_int64), _p(OV, C.c_uint64),
                      _p(F, C.c_double))
    return V, OV, F


def ga_migrate(pop, fit, n_migrants: int, island_base: int = 0):
    """One island-migration step (R16) on copies of pop [I][N][W] and fit [I][N]; returns (pop, fit)."""
    pop = np.array(pop, dtype=np.uint64, copy=True, order="C")
    fit = np.array(fit, dtype=np.float64, copy=True, order="C")
    I, N, W = pop.shape
    rc = lib().or_ga_migrate(W, N, I, n_migrants, island_base, _p(pop, C.c_uint64), _p(fit, C.c_double))
    if rc != 0:
        raise ValueError(f"or_ga_migrate rc={rc}")
    return pop, fit
