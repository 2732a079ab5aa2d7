"""C-ABI checks that need no GPU: the library loads, exports every symbol the
header declares, validates arguments, and its host-only Algorithm 1 matches the
literal oracle (exact rationals) decision for decision."""
import os
import random
import re

import numpy as np
import pytest

import oracle
from oracle.preempt import Request, preemption
from paper_conf_icpp_luoyww0023_b200 import split as S
from paper_conf_icpp_luoyww0023_b200 import workloads as wl
from split_testkit import ROOT


def _header_symbols():
    txt = open(os.path.join(ROOT, "include", "split_ga.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(split_[a-z_0-9]+)\s*\(", txt)))


def test_library_exports_every_header_symbol():
    syms = _header_symbols()
    assert len(syms) >= 15
    for s in syms:
        assert hasattr(S.lib(), s), s
    assert set(syms) == set(S.EXPORTED)


def test_strerror_and_defaults():
    assert S.lib().split_strerror(0) == b"ok"
    assert b"invalid" in S.lib().split_strerror(S.SPLIT_E_INVAL)
    d = S.split_ga_params_default()
    assert d["tournament_size"] == 4 and d["k_min"] == 2 and d["k_max"] == 32
    assert d["p_crossover"] == 0.9 and d["p_mutation"] == 0.2


@pytest.mark.parametrize("kw,code", [
    (dict(pop_size=255, n_elite=4), S.SPLIT_E_INVAL),            # (N - E) odd
    (dict(tournament_size=33), S.SPLIT_E_INVAL),
    (dict(k_min=5, k_max=4), S.SPLIT_E_INVAL),
    (dict(k_max=13), S.SPLIT_E_INVAL),                            # > n_ops
    (dict(n_elite=2000, pop_size=4000), S.SPLIT_E_INVAL),         # E > 1024
    (dict(p_mutation=1.5), S.SPLIT_E_INVAL),
    (dict(n_islands=2, islands_per_device=1), S.SPLIT_E_INVAL),   # spans ranks without comm
    (dict(n_islands=2, islands_per_device=2, migration_interval=5, n_migrants=0), S.SPLIT_E_INVAL),
])
def test_create_rejects_bad_params(kw, code):
    lat, ovh = wl.c1_chain()
    base = dict(pop_size=256, n_elite=4, k_min=2, k_max=12)
    base.update(kw)
    with pytest.raises(S.SplitError) as ei:
        S.SplitGA(lat, ovh, **base)
    assert ei.value.code == code


def test_create_range_guard():
    lat = np.full(12, 1 << 30, dtype=np.int64)          # T = 12 * 2^30 >= 2^32
    with pytest.raises(S.SplitError) as ei:
        S.SplitGA(lat, None, pop_size=256, n_elite=4, k_min=2, k_max=12)
    assert ei.value.code == S.SPLIT_E_RANGE
    with pytest.raises(S.SplitError) as ei:
        S.SplitGA(np.array([-1, 5], np.int64), None, pop_size=4, n_elite=0, k_min=1, k_max=2)
    assert ei.value.code == S.SPLIT_E_INVAL


def _rand_queue(rng, n, types=5, now=10_000_000):
    q = []
    for _ in range(n):
        ext = rng.randint(1, 300_000)
        q.append(Request(rng.randint(0, types), now - rng.randint(0, 5_000_000), ext, rng.randint(0, ext)))
    return q


def test_preempt_matches_literal_algorithm1():
    rng = random.Random(12345)
    now = 10_000_000
    for trial in range(3000):
        n = rng.randint(0, 40)
        q = _rand_queue(rng, n, types=rng.choice([1, 3, 20]))
        ext = rng.randint(1, 300_000)
        new = Request(rng.randint(0, 20), now - rng.randint(0, 1000), ext, ext if trial % 3 else rng.randint(0, ext))
        alpha = rng.choice([2.0, 4.0, 7.25, 20.0])
        ref = preemption(now, alpha, q, new)
        got = S.split_preempt_decide(now, alpha, [(t.type_id, t.arrival_ns, t.ext_ns, t.ext_left_ns) for t in q],
                                     (new.type_id, new.arrival_ns, new.ext_ns, new.ext_left_ns))
        assert got == ref, (trial, got, ref)


def test_preempt_ties_and_edges():
    now = 1000
    # equal Ext_left*Ext products stop the scan (line 13 uses >=)
    q = [(1, 0, 10, 10), (2, 0, 20, 5)]
    assert S.split_preempt_decide(now, 2.0, q, (3, now, 10, 10)) == 2
    assert preemption(now, 2.0, [Request(*x) for x in q], Request(3, now, 10, 10)) == 2
    assert S.split_preempt_decide(now, 2.0, [], (3, now, 10, 10)) == 0
    assert S.split_preempt_decide(now, 2.0, [(3, 0, 1000, 1000)], (3, now, 1, 1)) == 1   # same type: FIFO
    with pytest.raises(S.SplitError):
        S.split_preempt_decide(now, 0.0, q, (3, now, 10, 10))
    with pytest.raises(S.SplitError):
        S.split_preempt_decide(now, 2.0, q, (3, now, 10, 11))
    with pytest.raises(S.SplitError):
        S.split_preempt_decide(now, 2.0, [(1, 0, 0, 0)], (3, now, 10, 10))


def test_oracle_and_product_share_no_code():
    """The product never names oracle/, and oracle/ never names the product."""
    pkg = os.path.join(ROOT, "paper_conf_icpp_luoyww0023_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "split_oracle" not in txt, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c", ".h")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "paper_conf_icpp_luoyww0023_b200" not in txt.replace(
                "paper_conf_icpp_luoyww0023_b200/, include/split_ga.h", "").replace(
                "(``paper_conf_icpp_luoyww0023_b200``)", ""), f
            assert "split_ga.h\"" not in txt and "split_internal" not in txt, f


def test_qos_host_validation_without_gpu():
    # host-side argument checks run before any CUDA call (n_rep = 0: nothing to launch)
    import ctypes as C
    L = S.lib()
    blk = np.array([5, 5], dtype=np.int64)
    nb = np.array([2], dtype=np.uint32)
    al = np.array([2000], dtype=np.uint32)
    P64, P32 = C.POINTER(C.c_int64), C.POINTER(C.c_uint32)

    def el(uns, d=1, s=1, ref=None):
        u = None if uns is None else np.array(uns, dtype=np.int64).ctypes.data_as(P64)
        rf = None if ref is None else np.array(ref, dtype=np.int64).ctypes.data_as(P64)
        return L.split_qos_simulate_elastic(blk.ctypes.data_as(P64), nb.ctypes.data_as(P32), u, rf, 1, d, s,
                                            al.ctypes.data_as(P32), 1, 0, 0, None, None, None, None, None, 0, None)

    assert el([9]) == 0
    assert el([9], ref=[9]) == 0
    assert el(None) == S.SPLIT_E_INVAL                  # elastic needs the unsplit latencies
    assert el([0]) == S.SPLIT_E_RANGE                   # unsplit time out of [1, 2^32)
    assert el([1 << 32]) == S.SPLIT_E_RANGE
    assert el([9], ref=[0]) == S.SPLIT_E_RANGE          # latency reference out of [1, 2^32)
    base = lambda pol: L.split_qos_simulate(blk.ctypes.data_as(P64), nb.ctypes.data_as(P32), 1, pol,
                                            al.ctypes.data_as(P32), 1, 0, 0, None, None, None, None, None, 0, None)
    assert base(0) == 0 and base(1) == 0
    assert base(2) == S.SPLIT_E_INVAL                   # policy 2 only through split_qos_simulate_elastic
