"""Pins of the oracle GA's operators against the text of their readings, not
against the oracle itself (R7-R9, R16-R18, R22; P@21534-22160).

The paper leaves every operator detail open, so nothing it prints can pin the
GA trajectory.  What CAN pin it is the reading each operator follows.  Here
one generation is rebuilt in plain Python from those sentences alone --
Philox draws from ``oracle.philox`` (itself pinned by the Random123
known-answer vectors), integer arithmetic on Python ints -- and compared,
row by row, with what ``or_ga_run`` produced.  A plausible slip in the oracle
(a tie broken toward the higher index, the crossover halves swapped, the
mutation position off by the front, a repair that counts ranks from the top,
migrants written into the best slots, a Bernoulli compare with <=) fails
one of these tests.

R9  draw d of stream (id, gen, tag): lane d&3 of Philox4x32-10 at counter
    (id, gen, tag, d>>2), key (lo32 seed, hi32 seed); uniform in [0, m) is
    floor(u m / 2^32); Bernoulli(p) is u < floor(p 2^32).  Tags INIT=1
    SELECT=2 XOVER=3 (id = first child of the pair) MUTATE=4 REPAIR=5.
R7  s-way tournament with replacement: the winner is the max of (f, -index).
R8  children in pairs (c0 = E + 2q, c1 = c0 + 1) from the winners A (of c0)
    and B (of c1); with probability p_c one-point crossover at
    x = 1 + uniform(n-2): child0 = A's positions < x and B's >= x, child1 the
    complement; else copies.  Then, per child, with probability p_m flip the
    position front_skip + uniform(n-1-front_skip) (R22).
R17 repair: while popcount > k_max-1 clear the r-th set bit (ascending),
    r = uniform(c); while popcount < k_min-1 set the r-th unset position of
    [front_skip, n-2], r = uniform(n-1-front_skip-c).
R18 elites: the E best of generation g by (f desc, index asc) go to slots
    0..E-1 of g+1 in rank order.
R16 migration: each island's top-K by (f desc, index asc); an island sorts the
    foreign ones by (f desc, source island asc, rank asc) and writes the first
    K into its K worst slots, worst = (f asc, index desc), r-th worst <- r-th
    best.  Nothing else changes.
"""
import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl

INIT, SELECT, XOVER, MUTATE, REPAIR = 1, 2, 3, 4, 5


def draw(seed, gid, gen, tag, d):
    return oracle.philox((gid, gen, tag, d >> 2), (seed & 0xFFFFFFFF, seed >> 32))[d & 3]


def uniform(u, m):
    return (u * m) >> 32


def bern(u, p):
    thr = 0 if not p > 0 else (1 << 32 if p >= 1 else int(np.floor(p * 4294967296.0)))
    return u < thr


def row_int(row):
    return sum(int(w) << (64 * i) for i, w in enumerate(row))


def int_row(x, W):
    return np.array([(x >> (64 * i)) & ((1 << 64) - 1) for i in range(W)], dtype=np.uint64)


def one_generation(pop, fit, n, gen, seed, N, E, s, pc, pm, k_min, k_max, f=0):
    """Generation gen -> gen+1 of one island (ids = slots), from R7/R8/R9/R17/R18/R22."""
    order = sorted(range(N), key=lambda i: (-fit[i], i))
    rows = [None] * N
    for r in range(E):
        rows[r] = pop[order[r]]

    def winner(c):
        best = None
        for d in range(s):
            idx = uniform(draw(seed, c, gen, SELECT, d), N)
            if best is None or (fit[idx], -idx) > (fit[best], -best):
                best = idx
        return best

    mask_n = (1 << (n - 1)) - 1
    for c0 in range(E, N, 2):
        a, b = pop[winner(c0)], pop[winner(c0 + 1)]
        if bern(draw(seed, c0, gen, XOVER, 0), pc) and n >= 3:
            x = 1 + uniform(draw(seed, c0, gen, XOVER, 1), n - 2)
            lo = (1 << x) - 1
            kids = [(a & lo) | (b & ~lo & mask_n), (b & lo) | (a & ~lo & mask_n)]
        else:
            kids = [a, b]
        for h, ch in enumerate(kids):
            gid = c0 + h
            if bern(draw(seed, gid, gen, MUTATE, 0), pm):
                ch ^= 1 << (f + uniform(draw(seed, gid, gen, MUTATE, 1), n - 1 - f))
            d = 0
            cuts = [p for p in range(n - 1) if ch >> p & 1]
            while len(cuts) > k_max - 1:
                r = uniform(draw(seed, gid, gen, REPAIR, d), len(cuts))
                d += 1
                ch &= ~(1 << cuts.pop(r))
            while len(cuts) < k_min - 1:
                free = [p for p in range(f, n - 1) if not ch >> p & 1]
                r = uniform(draw(seed, gid, gen, REPAIR, d), n - 1 - f - len(cuts))
                d += 1
                ch |= 1 << free[r]
                cuts = [p for p in range(n - 1) if ch >> p & 1]
            rows[gid] = ch
    return rows


CASES = [
    # chain, N, E, s, p_c, p_m, k_min, k_max, front_skip
    ("ties", 64, 4, 4, 0.0, 0.0, 1, 12, 0),       # (a) pure selection on a tie-rich chain
    ("ties", 64, 2, 7, 0.0, 0.0, 1, 12, 0),
    ("ties", 40, 0, 1, 0.0, 0.0, 1, 12, 0),
    ("profile", 64, 4, 3, 1.0, 0.0, 1, 12, 0),    # (b) every pair crosses over, no repair
    ("profile", 96, 6, 4, 0.37, 0.61, 1, 12, 0),  # Bernoulli decisions both ways + mutation
    ("profile", 96, 4, 4, 1.0, 1.0, 4, 6, 0),     # (d) repair in both directions
    ("profile", 96, 4, 2, 1.0, 1.0, 5, 5, 3),     # fixed k with a guarded front (R22)
    ("resnet50_175", 128, 8, 4, 0.9, 0.2, 2, 32, 0),
    ("bert_base", 64, 4, 4, 1.0, 1.0, 6, 9, 150),  # W = 7: word boundaries in crossover and repair
]


def _chain(name):
    if name in ("ties", "profile"):
        return wl.c1_chain(overhead=name)
    return wl.chain(name)


@pytest.mark.parametrize("case", CASES, ids=[f"{c[0]}-N{c[1]}-s{c[3]}-pc{c[4]}-pm{c[5]}-k{c[6]}_{c[7]}" for c in CASES])
@pytest.mark.parametrize("seed", [5, (7 << 32) | 3])
def test_generation_rebuilt_from_the_readings(case, seed):
    name, N, E, s, pc, pm, k_min, k_max, f = case
    lat, ovh = _chain(name)
    n = len(lat)
    W = oracle.words(n)
    kw = dict(pop_size=N, n_elite=E, tournament_size=s, p_crossover=pc, p_mutation=pm, k_min=k_min,
              k_max=k_max, front_skip=f, want_population=True)
    prev = oracle.ga_run(lat, ovh, 0, seed, **kw)
    for gen in (0, 1):
        nxt = oracle.ga_run(lat, ovh, gen + 1, seed, **kw)
        pop = [row_int(r) for r in prev["population"][0]]
        fit = [float(x) for x in prev["fitness_all"][0]]
        want = one_generation(pop, fit, n, gen, seed, N, E, s, pc, pm, k_min, k_max, f)
        got = [row_int(r) for r in nxt["population"][0]]
        for c in range(N):
            assert got[c] == want[c], (gen, c)
        # each child's fitness is its row's Eq. 2 value (or_fitness, pinned separately)
        for c in range(E, N, max(1, N // 16)):
            st = oracle.fitness(lat, ovh, int_row(want[c], W), k_min, k_max)
            assert nxt["fitness_all"][0][c] == st["fitness"]
        prev = nxt


def test_selection_ties_go_to_the_lower_index():
    # constructed: on the all-ties chain (every k-block split of 12 equal ops with the same k and
    # block sizes has the same fitness) the tournament must pick the lowest drawn index among the
    # equal-fitness entrants; check that such ties actually occur and are resolved that way
    lat, ovh = wl.c1_chain(overhead="ties")
    N, E, s, seed = 64, 0, 8, 11
    r0 = oracle.ga_run(lat, ovh, 0, seed, pop_size=N, n_elite=E, tournament_size=s, p_crossover=0.0,
                       p_mutation=0.0, k_min=1, k_max=12, want_population=True)
    r1 = oracle.ga_run(lat, ovh, 1, seed, pop_size=N, n_elite=E, tournament_size=s, p_crossover=0.0,
                       p_mutation=0.0, k_min=1, k_max=12, want_population=True)
    fit = r0["fitness_all"][0]
    pop0, pop1 = r0["population"][0], r1["population"][0]
    ties = 0
    for c in range(N):
        ids = [uniform(draw(seed, c, 0, SELECT, d), N) for d in range(s)]
        fmax = max(fit[i] for i in ids)
        tied = sorted({i for i in ids if fit[i] == fmax})
        ties += len(tied) > 1
        assert np.array_equal(pop1[c], pop0[tied[0]])
    assert ties >= 5


def test_elites_are_the_best_in_rank_order():
    lat, ovh = wl.c1_chain(overhead="ties")            # many equal fitness values: index order decides
    N, E = 128, 16
    kw = dict(pop_size=N, n_elite=E, k_min=2, k_max=12, want_population=True)
    r0 = oracle.ga_run(lat, ovh, 0, 3, **kw)
    r1 = oracle.ga_run(lat, ovh, 1, 3, **kw)
    fit0 = r0["fitness_all"][0]
    order = sorted(range(N), key=lambda i: (-fit0[i], i))
    for r in range(E):
        assert np.array_equal(r1["population"][0][r], r0["population"][0][order[r]])
        assert r1["fitness_all"][0][r] == fit0[order[r]]


def _migrate_reference(pop, fit, K, base):
    I, N, _ = pop.shape
    tops = []
    for i in range(I):
        order = sorted(range(N), key=lambda c: (-fit[i][c], c))
        tops.append([(fit[i][order[r]], base + i, r, pop[i][order[r]].copy()) for r in range(K)])
    out_p, out_f = pop.copy(), fit.copy()
    for i in range(I):
        foreign = sorted((m for s in range(I) if s != i for m in tops[s]), key=lambda m: (-m[0], m[1], m[2]))
        worst = sorted(range(N), key=lambda c: (fit[i][c], -c))
        for r in range(min(K, len(foreign))):
            out_p[i][worst[r]] = foreign[r][3]
            out_f[i][worst[r]] = foreign[r][0]
    return out_p, out_f


@pytest.mark.parametrize("I,N,K,base", [(2, 16, 3, 0), (4, 32, 8, 4), (3, 12, 12, 0), (5, 40, 1, 2)])
def test_migration_replaces_exactly_the_worst_slots(I, N, K, base):
    rng = np.random.default_rng(I * 100 + K)
    W = 2
    pop = rng.integers(0, 1 << 62, size=(I, N, W), dtype=np.int64).astype(np.uint64)
    # few distinct values: ties inside an island, between islands and at the worst end
    fit = -rng.choice([0.5, 0.75, 0.75, 1.0, 1.25, 1.25, 1.25, 2.0], size=(I, N))
    got_p, got_f = oracle.ga_migrate(pop, fit, K, base)
    want_p, want_f = _migrate_reference(pop, fit, K, base)
    assert np.array_equal(got_p, want_p)
    assert np.array_equal(got_f, want_f)
    # nothing outside the K worst slots of each island changed
    for i in range(I):
        worst = set(sorted(range(N), key=lambda c: (fit[i][c], -c))[:K])
        for c in range(N):
            if c not in worst:
                assert np.array_equal(got_p[i][c], pop[i][c]) and got_f[i][c] == fit[i][c]


def test_migration_inside_the_ga_matches_the_step():
    # or_ga_run at a sync point == breed up to it, then exactly one migration step (R16)
    lat, ovh = wl.chain("resnet50_175")
    kw = dict(pop_size=64, n_elite=4, k_min=2, k_max=16, n_islands=3, n_migrants=5, want_population=True)
    no_mig = oracle.ga_run(lat, ovh, 3, 21, migration_interval=0, **kw)
    with_mig = oracle.ga_run(lat, ovh, 4, 21, migration_interval=3, **kw)
    # generation 3 of the migrating run: the islands of no_mig after one migration step; breeding
    # generation 3 -> 4 from it must give with_mig's generation 4; check the step through the
    # population it produces by re-running the reference migration on no_mig
    mp, mf = _migrate_reference(no_mig["population"], no_mig["fitness_all"], 5, 0)
    op, of = oracle.ga_migrate(no_mig["population"], no_mig["fitness_all"], 5, 0)
    assert np.array_equal(mp, op) and np.array_equal(mf, of)
    n = len(lat)
    for i in range(3):
        pop = [row_int(r) for r in op[i]]
        fit = [float(x) for x in of[i]]
        # island i breeds with ids i*N + slot: shift the ids through the seed-free formula
        want = _one_generation_island(pop, fit, n, 3, 21, i, 64, 4, 4, 0.9, 0.2, 2, 16)
        got = [row_int(r) for r in with_mig["population"][i]]
        assert got == want


def _one_generation_island(pop, fit, n, gen, seed, island, N, E, s, pc, pm, k_min, k_max):
    # one_generation with global ids island*N + slot (R9: id = island*N + local)
    off = island * N
    order = sorted(range(N), key=lambda i: (-fit[i], i))
    rows = [pop[order[r]] for r in range(E)] + [None] * (N - E)

    def winner(c):
        best = None
        for d in range(s):
            idx = uniform(draw(seed, off + c, gen, SELECT, d), N)
            if best is None or (fit[idx], -idx) > (fit[best], -best):
                best = idx
        return best

    mask_n = (1 << (n - 1)) - 1
    for c0 in range(E, N, 2):
        a, b = pop[winner(c0)], pop[winner(c0 + 1)]
        if bern(draw(seed, off + c0, gen, XOVER, 0), pc):
            x = 1 + uniform(draw(seed, off + c0, gen, XOVER, 1), n - 2)
            lo = (1 << x) - 1
            kids = [(a & lo) | (b & ~lo & mask_n), (b & lo) | (a & ~lo & mask_n)]
        else:
            kids = [a, b]
        for h, ch in enumerate(kids):
            gid = off + c0 + h
            if bern(draw(seed, gid, gen, MUTATE, 0), pm):
                ch ^= 1 << uniform(draw(seed, gid, gen, MUTATE, 1), n - 1)
            d = 0
            cuts = [p for p in range(n - 1) if ch >> p & 1]
            while len(cuts) > k_max - 1:
                r = uniform(draw(seed, gid, gen, REPAIR, d), len(cuts))
                d += 1
                ch &= ~(1 << cuts.pop(r))
            while len(cuts) < k_min - 1:
                free = [p for p in range(n - 1) if not ch >> p & 1]
                r = uniform(draw(seed, gid, gen, REPAIR, d), n - 1 - len(cuts))
                d += 1
                ch |= 1 << free[r]
                cuts = [p for p in range(n - 1) if ch >> p & 1]
            rows[c0 + h] = ch
    return rows


def test_init_follows_floyd_from_the_reading():
    # a1 (P@21534-21623, R9 INIT draws): k = k_min + uniform(k_max-k_min+1); then Floyd's sampling of
    # k-1 distinct positions of [f, n-2]: for j = m-(k-1) .. m-1 (m = n-1-f), r = uniform(j+1),
    # take f+r unless taken, else f+j
    lat, ovh = wl.chain("mobilenetv2")
    n = len(lat)
    N, f, seed = 96, 7, 99
    r = oracle.ga_run(lat, ovh, 0, seed, pop_size=N, n_elite=2, k_min=3, k_max=20, front_skip=f,
                      want_population=True)
    for c in range(N):
        d = 0
        k = 3 + uniform(draw(seed, c, 0, INIT, d), 18)
        d += 1
        m = n - 1 - f
        taken = set()
        for j in range(m - (k - 1), m):
            rr = uniform(draw(seed, c, 0, INIT, d), j + 1)
            d += 1
            taken.add(f + j if (f + rr) in taken else f + rr)
        assert row_int(r["population"][0][c]) == sum(1 << p for p in taken)


def test_bernoulli_threshold_is_strict():
    # R9: Bernoulli(p) is u < floor(p 2^32).  Construct p from the very draw it is compared with
    # (p = u0 / 2^32 is exact in binary64): then pair 0 must NOT cross over and child 0 must NOT
    # mutate, while any draw below the threshold does.
    lat, ovh = wl.c1_chain(overhead="profile")
    n = len(lat)
    seed, N = 17, 8
    u_x = draw(seed, 0, 0, XOVER, 0)
    u_m = draw(seed, 0, 0, MUTATE, 0)
    pc, pm = u_x / 4294967296.0, u_m / 4294967296.0
    kw = dict(pop_size=N, n_elite=0, tournament_size=2, p_crossover=pc, p_mutation=pm, k_min=1, k_max=12,
              want_population=True)
    r0 = oracle.ga_run(lat, ovh, 0, seed, **kw)
    r1 = oracle.ga_run(lat, ovh, 1, seed, **kw)
    pop = [row_int(r) for r in r0["population"][0]]
    fit = [float(x) for x in r0["fitness_all"][0]]
    want = one_generation(pop, fit, n, 0, seed, N, 0, 2, pc, pm, 1, 12)
    assert [row_int(r) for r in r1["population"][0]] == want
    # and the strict reading differs from "<=" on exactly this child
    assert not bern(u_x, pc) and not bern(u_m, pm)
    assert bern(u_x - 1, pc) and bern(u_m - 1, pm)
