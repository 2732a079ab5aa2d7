"""GPU parity of the f1 exact solvers through the C ABI:
split_exhaustive (all 2^(n-1) splits: canonical best, min V and argmin per k)
against the oracle's brute force (n <= 24), and split_dp_min_s2 against the
oracle's O(k n^2) DP (constant overhead) and against the exhaustive minima at
sizes the oracle cannot enumerate.  Every comparison is exact (integers and
bit-identical FP64)."""
import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def S():
    if not torch.cuda.is_available():
        pytest.fail("CUDA not available on a GPU test run")
    from paper_conf_icpp_luoyww0023_b200 import split
    return split


def _handle(S, lat, ovh, k_min, k_max):
    return S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=k_min, k_max=k_max)


def _check_against_brute(S, lat, ovh, k_min, k_max):
    n = len(lat)
    ref = oracle.brute(lat, ovh, k_min, k_max)
    with _handle(S, lat, ovh, k_min, k_max) as h:
        got = h.exhaustive(per_k=False)
    assert int(got["bits"][0]) == ref["bits"]
    assert np.float64(got["fitness"]).view(np.uint64) == np.float64(ref["fitness"]).view(np.uint64)
    assert got["k"] == ref["k"] and got["var_num"] == ref["var_num"]
    assert got["evaluations"] == 1 << (n - 1)
    # per-k minima over every k (handle with the full range)
    with _handle(S, lat, ovh, 1, n) as h:
        g2 = h.exhaustive(per_k=True)
    mv, am = g2["min_v_per_k"], g2["argmin_per_k"]
    for k in range(1, n + 1):
        assert mv[k] == ref["minV_per_k"][k], (k, mv[k], ref["minV_per_k"][k])
        assert int(am[k]) == int(ref["argminV_per_k"][k]), k


@pytest.mark.parametrize("kind", ["profile", "const", "zero", "ties"])
def test_c1_exhaustive_matches_brute(S, kind):
    """BASELINE configs[0]: 12-op chain, all 2^11 splits, GA range [2, 12]."""
    lat, ovh = wl.c1_chain(overhead=kind)
    _check_against_brute(S, lat, ovh, 2, 12)


@pytest.mark.parametrize("n,seed", [(2, 1), (3, 2), (5, 3), (7, 4), (8, 5), (13, 6), (17, 7), (20, 8), (24, 9)])
def test_random_chains_exhaustive_matches_brute(S, n, seed):
    # n - 1 <= 6 exercises the table-only path (no high part), larger n the Gray walk
    lat, ovh = wl.random_chain(n, seed, ovh_hi=200_000)
    k_lo = 1 if n < 4 else 2
    _check_against_brute(S, lat, ovh, k_lo, n)
    if n >= 5:
        # fixed block count (the paper's usage, R6)
        _check_against_brute(S, lat, ovh, 3, 3)


def test_exhaustive_ties_pick_smallest_bitset(S):
    lat = np.full(16, 1000, dtype=np.int64)            # many equal-fitness splits
    _check_against_brute(S, lat, None, 4, 4)


def test_dp_matches_oracle_constant_overhead(S):
    """C3: VGG-16 and MobileNetV2 shaped chains, k = 2..32, constant delta."""
    for name in ("vgg16", "mobilenetv2"):
        lat, _ = wl.chain(name)
        delta = int(0.05 * lat.sum())
        ovh = np.full(len(lat) - 1, delta, dtype=np.int64)
        kmax = min(32, len(lat))
        ref = oracle.dp(lat, delta, kmax)
        with _handle(S, lat, ovh, 1, kmax) as h:
            s2 = h.dp_min_s2(kmax)
        T = int(lat.sum())
        for k in range(1, kmax + 1):
            S1 = T + (k - 1) * delta
            V = (k * int(s2[k]) - S1 * S1)
            assert V == int(ref[k]), (name, k)


def test_dp_matches_exhaustive_minimum_at_scale(S):
    """n = 31 (2^30 splits, beyond the oracle's brute force): the exhaustive
    minimum V per k equals the DP optimum for a constant overhead."""
    lat, _ = wl.random_chain(31, 11)
    delta = int(0.04 * lat.sum())
    ovh = np.full(30, delta, dtype=np.int64)
    kmax = 31
    with _handle(S, lat, ovh, 1, kmax) as h:
        ex = h.exhaustive(per_k=True)
        s2 = h.dp_min_s2(kmax)
    T = int(lat.sum())
    for k in range(1, kmax + 1):
        S1 = T + (k - 1) * delta
        assert ex["min_v_per_k"][k] == k * int(s2[k]) - S1 * S1, k
    ref = oracle.dp(lat, delta, kmax)
    assert all(ex["min_v_per_k"][k] == ref[k] for k in range(1, kmax + 1))


def test_exhaustive_best_is_never_beaten_by_ga(S):
    """The GA best is a lower bound of the exact optimum (elitist search on the same fitness)."""
    lat, ovh = wl.random_chain(22, 5, ovh_hi=300_000)
    with _handle(S, lat, ovh, 2, 8) as h:
        ex = h.exhaustive()
    with S.SplitGA(lat, ovh, pop_size=512, n_elite=8, k_min=2, k_max=8) as g:
        r = g.run(40, 3)
    assert r["fitness"] <= ex["fitness"]


def test_exhaustive_rejects_large_n(S):
    lat = np.full(46, 10, dtype=np.int64)
    with _handle(S, lat, None, 2, 8) as h:
        with pytest.raises(S.SplitError):
            h.exhaustive()


@pytest.mark.parametrize("name", ["c1", "vgg16", "resnet50_175", "synthetic_1024"])
def test_heatmap2_matches_oracle(S, name):
    """f1 two-cut map (Fig. 2 analog): every entry of the (n-1)^2 map -- V, OV and the Eq. 2
    fitness bits -- equals the oracle's loop over or_fitness; synthetic_1024 (1023^2 entries,
    4096 CTAs) is compared on a strided sample of rows."""
    lat, ovh = wl.c1_chain() if name == "c1" else wl.chain(name)
    m = len(lat) - 1
    with S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=min(32, len(lat))) as h:
        V, OV, F = h.heatmap2()
        torch.cuda.synchronize()
    V, OV, F = V.cpu().numpy(), OV.cpu().numpy().view(np.uint64), F.cpu().numpy()
    if m <= 200:
        rV, rOV, rF = oracle.heatmap2(lat, ovh)
        assert np.array_equal(V, rV) and np.array_equal(OV, rOV)
        assert np.array_equal(F.view(np.uint64), rF.view(np.uint64))
    else:
        for a in list(range(0, m, 97)) + [m - 2, m - 1]:
            for b in range(m):
                if a > b:
                    assert V[a, b] == -1 and OV[a, b] == 0 and np.isneginf(F[a, b])
                    continue
                bits = np.zeros(oracle.words(len(lat)), np.uint64)
                for c in {a, b}:
                    bits[c >> 6] |= np.uint64(1 << (c & 63))
                st = oracle.fitness(lat, ovh, bits)
                assert V[a, b] == st["var_num"] and OV[a, b] == st["overhead"]
                assert np.float64(F[a, b]).view(np.uint64) == np.float64(st["fitness"]).view(np.uint64)


def test_heatmap2_guards(S):
    lat, ovh = wl.c1_chain()
    with S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=2) as h:
        with pytest.raises(S.SplitError) as e:
            h.heatmap2()
        assert e.value.code == S.SPLIT_E_INVAL
