"""GPU parity of split_ga_run (a1, a3-a9) against the oracle GA: the best
record, counters and the whole population (every row and every fitness bit)
after G generations must be identical.  All calls go through the C ABI."""
import math

import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ORACLE_KEYS = ("pop_size", "n_elite", "tournament_size", "p_crossover", "p_mutation", "k_min", "k_max",
               "front_skip", "stall_generations", "n_islands", "migration_interval", "n_migrants")


@pytest.fixture(scope="module")
def S():
    if not torch.cuda.is_available():
        pytest.fail("CUDA not available on a GPU test run")
    from paper_conf_icpp_luoyww0023_b200 import split
    return split


def _fbits(x):
    return np.asarray(x, np.float64).view(np.uint64)


def run_both(S, lat, ovh, G, seed, check_pop=True, **kw):
    kw.setdefault("islands_per_device", kw.get("n_islands", 1))
    h = S.SplitGA(lat, ovh, **kw)
    r = h.run(G, seed)
    okw = {k: v for k, v in kw.items() if k in ORACLE_KEYS}
    o = oracle.ga_run(lat, ovh, G, seed, want_population=check_pop, **okw)
    assert r["fitness"] == o["fitness"] or (math.isinf(r["fitness"]) and math.isinf(o["fitness"]))
    assert np.array_equal(r["bits"], o["bits"])
    for key in ("k", "var_num", "s1", "s2", "generation_found", "generations_run", "evaluations"):
        assert r[key] == o[key], (key, r[key], o[key])
    assert r["overhead_ns"] == o["overhead"]
    if check_pop:
        for i in range(kw.get("n_islands", 1)):
            bits, fit = h.population(i)
            assert np.array_equal(bits, o["population"][i]), f"island {i} rows differ"
            assert np.array_equal(_fbits(fit), _fbits(o["fitness_all"][i])), f"island {i} fitness differ"
    stats = h.last_run_stats()
    h.close()
    return r, o, stats


@pytest.mark.parametrize("seed", [1, 42, 20230807])
@pytest.mark.parametrize("G", [0, 1, 2, 7, 50])
def test_c1_trajectory(S, seed, G):
    lat, ovh = wl.c1_chain()
    run_both(S, lat, ovh, G, seed, pop_size=256, n_elite=4, k_min=2, k_max=12)


@pytest.mark.parametrize("k", list(range(2, 13)))
def test_c1_fixed_k_reaches_brute_force(S, k):
    lat, ovh = wl.c1_chain(overhead="const")
    r, o, _ = run_both(S, lat, ovh, 50, 42, pop_size=256, n_elite=4, k_min=k, k_max=k)
    b = oracle.brute(lat, ovh, k, k)
    assert r["fitness"] == b["fitness"] and int(r["bits"][0]) == b["bits"]


@pytest.mark.parametrize("name,N,E,G", [("resnet50_175", 4096, 82, 12), ("vgg16", 2048, 40, 20),
                                        ("bert_base", 2048, 40, 8), ("synthetic_1024", 1024, 20, 6),
                                        ("mobilenetv2", 8192, 1024, 6), ("gpt2", 256, 6, 4)])
def test_model_chains(S, name, N, E, G):
    lat, ovh = wl.chain(name)
    run_both(S, lat, ovh, G, 7, pop_size=N, n_elite=E, k_min=2, k_max=min(32, len(lat)))


def test_general_select_path_exercised(S):
    # a large random-ish population makes many children beat the worst elite early on,
    # forcing the radix top-E path; later generations use the candidate merge
    lat, ovh = wl.chain("resnet50_175")
    r, o, st = run_both(S, lat, ovh, 15, 3, pop_size=20000, n_elite=1024, k_min=2, k_max=32)
    assert st["general_selects"] >= 2 and st["fast_selects"] >= 1


@pytest.mark.parametrize("kw", [
    dict(pop_size=100, n_elite=0),
    dict(pop_size=64, n_elite=64),
    dict(pop_size=130, n_elite=2, tournament_size=1),
    dict(pop_size=130, n_elite=2, tournament_size=32),
    dict(pop_size=128, n_elite=8, p_crossover=0.0, p_mutation=0.0, k_min=1, k_max=105),
    dict(pop_size=128, n_elite=8, p_crossover=1.0, p_mutation=1.0),
    dict(pop_size=128, n_elite=8, k_min=5, k_max=5, front_skip=60),
    dict(pop_size=256, n_elite=8, k_min=3, k_max=9, front_skip=90, p_mutation=1.0),
    dict(pop_size=128, n_elite=8, k_min=1, k_max=3),
])
def test_edge_parameters(S, kw):
    lat, ovh = wl.chain("mobilenetv2")
    base = dict(k_min=2, k_max=32)
    base.update(kw)
    run_both(S, lat, ovh, 9, 11, **base)


def test_stall_termination(S):
    lat, ovh = wl.c1_chain()
    r, o, _ = run_both(S, lat, ovh, 500, 1, pop_size=256, n_elite=4, k_min=2, k_max=12, stall_generations=15)
    assert r["generations_run"] < 500


def test_zero_chain_ties(S):
    lat, ovh = wl.c1_chain(overhead="ties")
    run_both(S, lat, ovh, 30, 5, pop_size=256, n_elite=4, k_min=2, k_max=12)


@pytest.mark.parametrize("M,stall", [(3, 0), (0, 0), (4, 8), (2, 3)])
def test_local_islands_with_migration(S, M, stall):
    lat, ovh = wl.chain("resnet50_175")
    run_both(S, lat, ovh, 13, 77, pop_size=128, n_elite=4, k_min=2, k_max=16, n_islands=4,
             migration_interval=M, n_migrants=4 if M else 0, stall_generations=stall)


def test_islands_eight_large_migrants(S):
    lat, ovh = wl.chain("bert_base")
    run_both(S, lat, ovh, 10, 9, pop_size=512, n_elite=16, k_min=2, k_max=32, n_islands=8,
             migration_interval=2, n_migrants=64)


def test_c2_full_size_first_generations(S):
    """C2 at the size bench.py runs (n = 175, N = 65,536, E = 1024): the first
    generations are compared bit for bit with the oracle."""
    lat, ovh = wl.chain("resnet50_175")
    run_both(S, lat, ovh, 4, 20230807, pop_size=65536, n_elite=1024, k_min=2, k_max=32)


def test_c2_full_run_invariants(S):
    lat, ovh = wl.chain("resnet50_175")
    h = S.SplitGA(lat, ovh, pop_size=65536, n_elite=1024, k_min=2, k_max=32)
    r = h.run(500, 1)
    bits, fit = h.population(0)
    h.close()
    assert r["generations_run"] == 500 and r["evaluations"] == 65536 + 500 * 64512
    assert np.all(np.diff(fit[:1024]) <= 0)          # elites in rank order
    assert r["fitness"] >= fit.max()
    # the reported best re-evaluates to itself on the oracle
    s = oracle.fitness(lat, ovh, r["bits"], 2, 32)
    assert s["fitness"] == r["fitness"] and s["var_num"] == r["var_num"] and s["k"] == r["k"]
    assert r["expected_wait_ns"] == pytest.approx(s["s2"] / (2 * s["s1"]))


def test_islands_through_nccl_communicator(S):
    """The island exchange through a (1-rank) NCCL communicator: same trajectory
    as the oracle's serial islands (the all-gathers run in NCCL)."""
    uid = S.split_comm_unique_id()
    comm = S.split_comm_init(uid, 0, 1, 0)
    try:
        lat, ovh = wl.chain("resnet50_175")
        kw = dict(pop_size=256, n_elite=8, k_min=2, k_max=16, n_islands=4, islands_per_device=4,
                  migration_interval=3, n_migrants=8)
        h = S.SplitGA(lat, ovh, comm=comm, **kw)
        r = h.run(10, 5)
        pops = [h.population(i) for i in range(4)]
        h.close()
    finally:
        S.split_comm_destroy(comm)
    o = oracle.ga_run(lat, ovh, 10, 5, want_population=True,
                      **{k: v for k, v in kw.items() if k in ORACLE_KEYS})
    assert r["fitness"] == o["fitness"] and np.array_equal(r["bits"], o["bits"])
    assert r["generation_found"] == o["generation_found"]
    for i in range(4):
        assert np.array_equal(pops[i][0], o["population"][i])


def test_large_population_several_chunks_per_warp(S):
    """N = 262,144 on the BERT-base chain (W = 7, register rows of 8 words): every
    worker warp breeds several 32-child chunks per generation (the large-N loop
    that the C4-shaped bench island runs), compared bit for bit."""
    lat, ovh = wl.chain("bert_base")
    run_both(S, lat, ovh, 2, 42, pop_size=262144, n_elite=1024, k_min=2, k_max=32)


def test_hbm_regime_island_first_generation(S):
    """The bench's `ga_hbm_regime` configuration itself (N = 4,194,304, W = 7):
    generation 0 and one transition, whole population bit for bit."""
    lat, ovh = wl.chain("bert_base")
    run_both(S, lat, ovh, 1, 77, pop_size=1 << 22, n_elite=1024, k_min=2, k_max=32)


def test_set_chain_matches_fresh_handle(S):
    """split_ga_set_chain on a live handle == a handle created with that chain ==
    the oracle; bad chains are rejected like split_ga_create rejects them."""
    lat1, ovh1 = wl.chain("resnet50_175")
    lat2, ovh2 = wl.chain("resnet50_175", overhead="const")
    lat2 = lat2[::-1].copy()
    kw = dict(pop_size=4096, n_elite=82, k_min=2, k_max=32)
    with S.SplitGA(lat1, ovh1, **kw) as h:
        h.run(5, 1)
        h.set_chain(lat2, ovh2)
        r = h.run(12, 7)
        bits, fit = h.population(0)
        with pytest.raises(S.SplitError) as e:
            h.set_chain(-lat2, ovh2)
        assert e.value.code == S.SPLIT_E_INVAL
    o = oracle.ga_run(lat2, ovh2, 12, 7, want_population=True, **kw)
    assert r["fitness"] == o["fitness"] and np.array_equal(r["bits"], o["bits"])
    assert np.array_equal(bits, o["population"][0])
    assert np.array_equal(_fbits(fit), _fbits(o["fitness_all"][0]))


@pytest.mark.parametrize("name", ["c1", "vgg16"])
def test_k_sweep_eq1_choice(S, name):
    """f3 (R21): split_k_sweep == one oracle fixed-k GA per k, and with a
    constant per-cut overhead (S1 and OV fixed per k) each k's best reaches the
    exact minimum S2 of the DP, so the chosen k is the exact argmin over k of
    J(k) = S2/(2 S1) + OV (Eq. 1's wait plus the added latency, P@18542-18830)
    computed here in rationals from the oracle DP -- an interior k (3) on both
    chains, not the end of the range."""
    from fractions import Fraction
    if name == "c1":
        lat, ovh = wl.c1_chain(overhead="const")
        kw, G, k_hi = dict(pop_size=256, n_elite=4, k_min=2, k_max=12), 50, 12
    else:
        lat, _ = wl.chain("vgg16")
        ovh, _ = wl.constant_overhead(lat)
        kw, G, k_hi = dict(pop_size=4096, n_elite=64, k_min=2, k_max=16), 40, 16
    delta = int(ovh[0])
    with S.SplitGA(lat, ovh, **kw) as h:
        kb, res = h.k_sweep(2, k_hi, G, 42)
        r_after = h.run(3, 1)                       # the handle's own k range is restored
    o_after = oracle.ga_run(lat, ovh, 3, 1, **kw)
    assert r_after["fitness"] == o_after["fitness"]
    V = oracle.dp(lat, delta, k_hi)
    T = int(lat.sum())
    J = {}
    for r in res:
        k = r["k"]
        o = oracle.ga_run(lat, ovh, G, 42, **{**kw, "k_min": k, "k_max": k})
        assert r["fitness"] == o["fitness"] and r["var_num"] == o["var_num"]
        assert r["s1"] == o["s1"] and r["s2"] == o["s2"] and r["overhead_ns"] == o["overhead"]
        assert r["expected_wait_ns"] == o["s2"] / (2.0 * o["s1"])
        assert r["cost_ns"] == r["expected_wait_ns"] + float(o["overhead"])
        S1 = T + (k - 1) * delta
        assert (int(V[k]) + S1 * S1) % k == 0
        s2_min = (int(V[k]) + S1 * S1) // k
        assert r["s2"] == s2_min                    # the GA reached the DP optimum for this k
        J[k] = Fraction(s2_min, 2 * S1) + (k - 1) * delta
    k_star = min(J, key=lambda k: (J[k], k))
    assert 2 < k_star < k_hi                        # the criterion has an interior optimum here
    assert kb == k_star


def test_c2_full_length_parity(S):
    """The bench step itself (C2: n = 175, N = 65,536, E = 1024, s = 4, 500 generations):
    final population, every fitness bit, the best record and the counters against the
    oracle GA (about half a minute of one CPU core)."""
    lat, ovh = wl.chain("resnet50_175")
    run_both(S, lat, ovh, 500, 1, pop_size=65536, n_elite=1024, tournament_size=4, p_crossover=0.9,
             p_mutation=0.2, k_min=2, k_max=32)


def test_c4_shaped_batched_islands(S):
    """C4's island model shape (BERT-base chain, W = 7; top-64 migration every 10
    generations) with 8 islands of 65,536 batched on one GPU, 30 generations: every
    island bit for bit against the oracle's serial islands."""
    lat, ovh = wl.chain("bert_base")
    run_both(S, lat, ovh, 30, 8, pop_size=65536, n_elite=1024, k_min=2, k_max=32, n_islands=8,
             migration_interval=10, n_migrants=64)


@pytest.mark.parametrize("N,K,I,M", [(8192, 32, 4, 3), (65536, 200, 3, 4), (3000, 16, 5, 2)])
def test_sync_point_selection_paths(S, N, K, I, M):
    """The sync point's selections take different paths by size (one-warp sort for
    <= 512 entries, the radix select beyond; the collection threshold from a
    two-level warp sort of the sample or the radix select): island sizes between the
    whole-island sort and C4's 65,536, and a K whose collection exceeds one warp's
    sort, all bit for bit against the oracle's serial islands."""
    lat, ovh = wl.chain("vgg16")
    run_both(S, lat, ovh, 3 * M + 1, 11, pop_size=N, n_elite=16, k_min=2, k_max=12, n_islands=I,
             migration_interval=M, n_migrants=K)


def test_comm_layout_checked_at_create(S):
    """A communicator of world 1 cannot host islands of another layout (advisor: the
    all-gathers would write past the buffers); the device must match too."""
    uid = S.split_comm_unique_id()
    comm = S.split_comm_init(uid, 0, 1, 0)
    try:
        lat, ovh = wl.chain("vgg16")
        for bad in (dict(n_islands=2, islands_per_device=1, island_id=0),
                    dict(n_islands=2, islands_per_device=1, island_id=1)):
            with pytest.raises(S.SplitError) as e:
                S.SplitGA(lat, ovh, comm=comm, pop_size=64, n_elite=2, migration_interval=2, n_migrants=2, **bad)
            assert e.value.code == S.SPLIT_E_INVAL
        with S.SplitGA(lat, ovh, comm=comm, pop_size=64, n_elite=2, n_islands=2, islands_per_device=2,
                       migration_interval=2, n_migrants=2) as h:
            h.run(3, 1)
    finally:
        S.split_comm_destroy(comm)
