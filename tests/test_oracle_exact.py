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
