"""Pins for the CPU oracle's core arithmetic (Philox, dexp, Eq. 2 fitness, Eq. 1).

Every check compares the oracle with something other than itself: published
known-answer vectors, a 300-bit mpmath evaluation, closed forms, numpy's
population standard deviation of an independently derived block list, and
exact rational identities.
"""
import math
from fractions import Fraction

import mpmath
import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl
from split_testkit import golden_rows

mpmath.mp.prec = 300


def _golden(name):
    return golden_rows(name)


def test_philox_known_answers():
    rows = _golden("philox_kat.txt")
    assert len(rows) == 3
    for r in rows:
        v = [int(x, 16) for x in r]
        assert oracle.philox(v[0:4], v[4:6]) == tuple(v[6:10])


def _ulp_err(got: float, z: float) -> float:
    true = mpmath.exp(mpmath.mpf(z))
    ulp = math.ulp(float(true))
    return float(abs(mpmath.mpf(got) - true) / ulp)


def test_dexp_within_one_ulp():
    rng = np.random.default_rng(5)
    zs = list(rng.uniform(-1, 3, 3000)) + list(rng.uniform(-1, 700, 1000))
    zs += [-1.0, -0.5, 0.0, 0.34657359027997264, -0.34657359027997264, 1.0, 2.0, 700.0, 709.0]
    worst = max(_ulp_err(oracle.dexp(z), z) for z in zs)
    assert worst < 1.0, worst


def test_dexp_special_values():
    # RN(1/e): the k=1 value of each Eq. 2 term
    assert oracle.dexp(-1.0) == float.fromhex("0x1.78b56362cef38p-2")
    assert oracle.dexp(0.0) == 1.0
    assert oracle.dexp(711.0) == math.inf


def test_fitness_unsplit_is_minus_two_over_e():
    rows = {r[0]: r[1] for r in _golden("paper_numbers.txt")}
    lat, ovh = wl.random_chain(20, 3, ovh_hi=5000)
    s = oracle.fitness(lat, ovh, np.zeros(1, np.uint64), k_min=1)
    assert s["k"] == 1 and s["var_num"] == 0 and s["overhead"] == 0
    assert s["fitness"] == float.fromhex(rows["fitness_unsplit"])


def _blocks(lat, ovh, cuts):
    """Block times by np.split of the latency list; the block after cut p pays ovh[p]."""
    parts = np.split(np.asarray(lat, dtype=np.int64), [c + 1 for c in cuts])
    t = [int(p.sum()) for p in parts]
    for j, c in enumerate(cuts):
        t[j + 1] += int(ovh[c])
    return t


def test_two_block_closed_form():
    lat, ovh = wl.random_chain(30, 4, ovh_hi=20000)
    for c in range(29):
        bits = wl.pack_positions([[c]], 30)[0]
        s = oracle.fitness(lat, ovh, bits, k_min=1)
        t1 = int(lat[: c + 1].sum())
        t2 = int(lat[c + 1:].sum()) + int(ovh[c])
        assert s["k"] == 2
        assert s["var_num"] == (t1 - t2) ** 2
        assert s["overhead"] == ovh[c]


def test_constant_chain_even_cuts_zero_variance():
    n, k = 24, 4
    lat = np.full(n, 777, dtype=np.int64)
    cuts = [n // k * j - 1 for j in range(1, k)]
    bits = wl.pack_positions([cuts], n)[0]
    s = oracle.fitness(lat, np.zeros(n - 1, np.int64), bits, k_min=1)
    assert s["k"] == k and s["var_num"] == 0
    # sigma = 0 => the first Eq. 2 term is e^{-1}; OV = 0 => so is the second
    assert s["fitness"] == -2 * oracle.dexp(-1.0)


def test_constant_overhead_shift_keeps_variance():
    # adding the same delta to every block but the first changes t_1 relative to the
    # others; adding delta to lat[0] as well shifts ALL blocks by delta: V unchanged
    lat, _ = wl.random_chain(40, 8)
    rng = np.random.default_rng(1)
    for _ in range(20):
        cuts = sorted(rng.choice(39, size=rng.integers(1, 10), replace=False).tolist())
        bits = wl.pack_positions([cuts], 40)[0]
        base = oracle.fitness(lat, np.zeros(39, np.int64), bits, k_min=1)
        delta = 12345
        lat2 = lat.copy()
        lat2[0] += delta
        shifted = oracle.fitness(lat2, np.full(39, delta, np.int64), bits, k_min=1)
        assert shifted["var_num"] == base["var_num"]


def test_fitness_matches_numpy_std_and_high_precision_eq2():
    for name in ["resnet50_175", "bert_base", "vgg16", "synthetic_1024"]:
        lat, ovh = wl.chain(name)
        n = len(lat)
        T = int(lat.sum())
        pop = wl.sparse_population(n, 60, seed=7, k_lo=1, k_hi=40)
        for row in pop:
            cuts = [p for p in range(n - 1) if (int(row[p >> 6]) >> (p & 63)) & 1]
            s = oracle.fitness(lat, ovh, row, k_min=1)
            t = _blocks(lat, ovh, cuts)
            k = len(t)
            assert s["k"] == k
            assert s["s1"] == sum(t) and s["s2"] == sum(x * x for x in t)
            assert s["overhead"] == sum(int(ovh[c]) for c in cuts)
            # population sigma (ddof=0) — reading R1
            sigma_np = float(np.std(np.array(t, dtype=np.float64)))
            sigma_or = math.sqrt(s["var_num"]) / k
            assert sigma_or == pytest.approx(sigma_np, rel=1e-9, abs=1e-6)
            # Eq. 2 evaluated at 300 bits from the block list
            sig = mpmath.sqrt(mpmath.mpf(sum((mpmath.mpf(x) - mpmath.mpf(sum(t)) / k) ** 2 for x in t)) / k)
            ovr = mpmath.mpf(s["overhead"]) / T
            f_true = -(mpmath.exp(sig / T - 1) + mpmath.exp(ovr / k - 1))
            assert abs(mpmath.mpf(s["fitness"]) - f_true) <= 4 * math.ulp(float(f_true))


def test_eq1_identity_exact():
    """Eq. 1 (P@17448-17827): 1/2 sum t^2 / sum t == 1/2 (sigma^2/tbar + tbar), in rationals."""
    lat, ovh = wl.chain("googlenet")
    n = len(lat)
    for row in wl.sparse_population(n, 50, seed=3, k_lo=1, k_hi=20):
        s = oracle.fitness(lat, ovh, row, k_min=1)
        k, S1, S2, V = s["k"], s["s1"], s["s2"], s["var_num"]
        lhs = Fraction(S2, 2 * S1)
        sigma2 = Fraction(V, k * k)
        tbar = Fraction(S1, k)
        assert lhs == Fraction(1, 2) * (sigma2 / tbar + tbar)


def test_eq1_expected_wait_by_integration():
    """The expected wait of Eq. 1's integral, integrated numerically, equals S2/(2 S1)."""
    lat, ovh = wl.chain("yolov2")
    n = len(lat)
    row = wl.sparse_population(n, 1, seed=9, k_lo=5, k_hi=5)[0]
    s = oracle.fitness(lat, ovh, row, k_min=1)
    cuts = [p for p in range(n - 1) if (int(row[p >> 6]) >> (p & 63)) & 1]
    t = _blocks(lat, ovh, cuts)
    ends = np.cumsum(t)
    total = ends[-1]
    arrive = (np.arange(200000) + 0.5) * total / 200000
    wait = ends[np.searchsorted(ends, arrive, side="right")] - arrive
    assert float(wait.mean()) == pytest.approx(s["s2"] / (2 * s["s1"]), rel=1e-6)


def test_padding_bits_ignored_and_k_range():
    lat, ovh = wl.random_chain(70, 11, ovh_hi=1000)   # n-1 = 69 positions -> W = 2, 59 padding bits
    row = wl.pack_positions([[3, 40, 68]], 70)[0]
    s = oracle.fitness(lat, ovh, row, k_min=1)
    row2 = row.copy()
    row2[1] |= np.uint64(0xFFFFFFFFFFFFFFFF) << np.uint64(5)
    s2 = oracle.fitness(lat, ovh, row2, k_min=1)
    assert s == s2
    assert oracle.fitness(lat, ovh, row, k_min=5)["fitness"] == -math.inf
    assert oracle.fitness(lat, ovh, row, k_min=1, k_max=3)["fitness"] == -math.inf
    assert oracle.fitness(lat, ovh, row, k_min=4, k_max=4)["fitness"] > -math.inf


def test_batch_equals_single():
    lat, ovh = wl.chain("mobilenetv2")
    pop = wl.sparse_population(len(lat), 100, seed=2)
    fb = oracle.fitness_batch(lat, ovh, pop, 2, 32)
    for i, row in enumerate(pop):
        assert fb[i] == oracle.fitness(lat, ovh, row, 2, 32)["fitness"]
