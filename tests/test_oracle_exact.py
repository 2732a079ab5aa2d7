"""Pins for the oracle's exact solvers: brute force vs the O(k n^2) DP, and the
paper's candidate count (§2.2, P@9788-10019)."""
import math

import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl
from split_testkit import golden_rows


def test_paper_candidate_count_resnet50():
    rows = {r[0]: int(r[1]) for r in golden_rows("paper_numbers.txt") if r[0].startswith("resnet50")}
    n = rows["resnet50_ops"]
    # "3 blocks" in the text is 3 cut points (4 blocks) — reading R14
    assert oracle.count_fixed_k(n, 4) == rows["resnet50_candidates_3cuts"] == math.comb(n - 1, 3)


@pytest.mark.parametrize("n,k", [(12, 1), (12, 2), (12, 12), (20, 6), (37, 3), (105, 3)])
def test_count_fixed_k_binomial(n, k):
    assert oracle.count_fixed_k(n, k) == math.comb(n - 1, k - 1)


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
@pytest.mark.parametrize("delta", [0, 37, 500])
def test_brute_force_equals_dp(seed, delta):
    n = 11 + seed % 3
    lat, _ = wl.random_chain(n, 100 + seed, lo=1, hi=2000)
    ovh = np.full(n - 1, delta, dtype=np.int64)
    b = oracle.brute(lat, ovh)
    vstar = oracle.dp(lat, delta, n)
    for k in range(1, n + 1):
        assert b["minV_per_k"][k] == vstar[k], (k, b["minV_per_k"][k], vstar[k])
    # the global Eq. 2 optimum over a k range is the best of the per-k optima
    T = int(lat.sum())
    for kmin, kmax in [(2, n), (2, 4), (3, 3)]:
        bk = oracle.brute(lat, ovh, kmin, kmax)
        f_dp = max(oracle.fitness_from(k, int(vstar[k]), (k - 1) * delta, T) for k in range(kmin, kmax + 1))
        assert bk["fitness"] == f_dp


def test_unsplit_wins_without_k_floor():
    # reading R6: with k = 1 allowed, both Eq. 2 terms take their minimum e^-1
    lat, ovh = wl.c1_chain()
    b = oracle.brute(lat, ovh, 1, 12)
    assert b["k"] == 1 and b["bits"] == 0


def test_brute_canonical_tie_break():
    # tie-rich chain: all ops 1000 ns, no overhead; k = 3 even splits 4|4|4 are unique,
    # but k = 5 has several equal-V splits; the canonical best is the smallest bitset
    lat, ovh = wl.c1_chain(overhead="ties")
    b = oracle.brute(lat, ovh, 5, 5)
    cands = []
    for m in range(1 << 11):
        if bin(m).count("1") != 4:
            continue
        s = oracle.fitness(lat, ovh, np.array([m], np.uint64), 5, 5)
        cands.append((-s["fitness"], m))
    best = min(cands)
    assert b["bits"] == best[1]
    ties = [m for f, m in cands if f == best[0]]
    assert len(ties) > 1 and b["bits"] == min(ties)


def test_dp_constant_chain_even_split():
    lat = np.full(60, 100, dtype=np.int64)
    v = oracle.dp(lat, 0, 10)
    for k in (1, 2, 3, 4, 5, 6, 10):
        assert v[k] == 0          # 60 divisible by k
    assert v[7] > 0


@pytest.mark.parametrize("name", ["c1", "vgg16"])
def test_heatmap2_pins(name):
    """Two-cut map (Fig. 2 analog, P@11560-12128): each entry's sigma is numpy's population
    std of the explicit block-time list (built here from cumulative sums, not from the oracle),
    the overhead is the sum of the two cuts' overheads, the minimum over the upper triangle is
    brute force's minimum V for 3 blocks and over the diagonal the one for 2 blocks."""
    if name == "c1":
        lat, ovh = wl.c1_chain()
    else:
        lat, ovh = wl.chain("vgg16")
    n = len(lat)
    m = n - 1
    V, OV, F = oracle.heatmap2(lat, ovh)
    cs = np.concatenate([[0], np.cumsum(lat)])
    T = int(cs[-1])
    rng = np.random.default_rng(1)
    pairs = [(a, b) for a in range(m) for b in range(a, m)]
    for a, b in (pairs if len(pairs) < 100 else [pairs[i] for i in rng.choice(len(pairs), 120, replace=False)]):
        cuts = [a] if a == b else [a, b]
        ends = [int(cs[c + 1]) for c in cuts] + [T]
        starts = [0] + [int(cs[c + 1]) for c in cuts]
        t = np.array([e - s for s, e in zip(starts, ends)], dtype=np.float64)
        t[1:] += [float(ovh[c]) for c in cuts]
        k = len(t)
        assert math.isclose(math.sqrt(V[a, b]) / k, float(np.std(t)), rel_tol=1e-12, abs_tol=1e-6)
        assert int(OV[a, b]) == sum(int(ovh[c]) for c in cuts)
        x = math.sqrt(V[a, b]) / (k * T)
        y = (int(OV[a, b]) / T) / k
        assert math.isclose(F[a, b], -(math.exp(x - 1) + math.exp(y - 1)), rel_tol=1e-14)
    lower = np.tril_indices(m, -1)
    assert (V[lower] == -1).all() and (OV[lower] == 0).all() and np.isneginf(F[lower]).all()
    if n <= 20:
        b = oracle.brute(lat, ovh)
        iu = np.triu_indices(m, 1)
        assert V[iu].min() == b["minV_per_k"][3]
        assert np.diag(V).min() == b["minV_per_k"][2]
