"""Pins for the f2 QoS simulator oracle (oracle/qos.py, R20).

Checks against what the paper's scheduling semantics and queueing theory fix,
not against the oracle itself: a worked two-model example computed by hand
from §3.4 (preemption only between blocks, Algorithm 1's pass rule), Lindley's
recursion for a FIFO single-server queue, the same-type rule (a request never
passes one of its own task: Algorithm 1 line 6), and work conservation (the
executor's busy periods do not depend on the order it serves requests in).
"""
import numpy as np

from oracle import qos
from paper_conf_icpp_luoyww0023_b200 import workloads as wl


def test_single_request_runs_in_isolation():
    for pol in (qos.FIFO, qos.ALG1):
        assert qos.simulate([[3, 4, 5]], [100], [0], pol) == [12]


def test_worked_example_preemption_between_blocks():
    # L = 3 blocks of 5 (Ext 15) arrives at 0; S = one block of 2 arrives at 1.
    # Algorithm 1 at t = 1: Q = [L with Ext_left 10 (blocks 2, 3 not started)];
    # Ext_left(L) Ext(L) = 150 > Ext_left(S) Ext(S) = 4 -> S passes L and runs
    # at the next block boundary (5..7); L resumes 7..17.
    blocks = [[5, 5, 5], [2]]
    assert qos.simulate(blocks, [0, 1], [0, 1], qos.ALG1) == [17, 6]
    # FIFO: S waits for all of L
    assert qos.simulate(blocks, [0, 1], [0, 1], qos.FIFO) == [15, 16]
    # unsplit L (one block): no boundary before 15 under either policy
    assert qos.simulate([[15], [2]], [0, 1], [0, 1], qos.ALG1) == [15, 16]
    # statistics: RR = 17/15 and 6/2; alpha = 2 -> only S (RR 3) violates
    viol, rs, rq = qos.stats(blocks, [0, 1], [17, 6], [1000, 2000, 3000])
    assert viol == [2, 1, 0]
    assert rs == 17 / 15 + 3.0
    assert rq == (17 / 15) ** 2 + 9.0


def test_arrival_at_block_end_is_inserted_first():
    # S arrives exactly when L's first block ends: it is queued before the
    # executor picks the next block, so it runs 5..7
    assert qos.simulate([[5, 5, 5], [2]], [0, 5], [0, 1], qos.ALG1) == [17, 2]


def test_fifo_single_type_is_lindley():
    arr, _ = wl.qos_requests(3, 300, 9_000_000, 1, seed=5)
    blocks = [[2_000_000, 3_000_000, 4_000_000]]
    S = sum(blocks[0])
    for r in range(3):
        a = [int(x) for x in arr[r]]
        got = qos.simulate(blocks, a, [0] * len(a), qos.FIFO)
        w = 0
        for i in range(len(a)):
            if i:
                w = max(0, w + S - (a[i] - a[i - 1]))
            assert got[i] == w + S


def test_same_type_never_passes_and_busy_periods_are_policy_free():
    arr, ty = wl.qos_requests(2, 250, 7_000_000, 4, seed=9)
    blocks = wl.random_blocks(4, seed=3, k_hi=5, lo=500_000, hi=6_000_000)
    ext = [sum(b) for b in blocks]
    for r in range(2):
        a = [int(x) for x in arr[r]]
        t = [int(x) for x in ty[r]]
        f = qos.simulate(blocks, a, t, qos.FIFO)
        g = qos.simulate(blocks, a, t, qos.ALG1)
        # completion instants: every request finishes no earlier than arrival + Ext
        for i in range(len(a)):
            assert f[i] >= ext[t[i]] and g[i] >= ext[t[i]]
        # work conservation: the last completion (end of the last busy period) is the same
        assert max(a[i] + f[i] for i in range(len(a))) == max(a[i] + g[i] for i in range(len(a)))
        # one type only: Algorithm 1 never reorders (line 6) -> identical to FIFO
        same = [0] * len(a)
        assert qos.simulate(blocks, a, same, qos.ALG1) == qos.simulate(blocks, a, same, qos.FIFO)


# ---- f4 elastic splitting (ELASTIC, R23; §3.3 P@22612-23675) ----

def test_elastic_worked_examples_by_hand():
    # L: 3 blocks of 5 (Ext 15), unsplit T = 13 (no cut overheads); S: one block of 2 (T = 2)
    blocks, uns = [[5, 5, 5], [2]], [13, 2]
    big = 1 << 30
    # density: S arrives to 1 pending request (L, blocks 2 and 3 not started).
    # d_max = 1 -> splitting off for S: unsplit, at the tail, runs after L (15..17)
    assert qos.simulate(blocks, [0, 1], [0, 1], qos.ELASTIC, uns, 1, big) == [15, 16]
    # d_max = 2 -> S is split and passes L (Algorithm 1), as under ALG1
    assert qos.simulate(blocks, [0, 1], [0, 1], qos.ELASTIC, uns, 2, big) == [17, 6]
    # same type: a second L arrives while L is pending.  s_max = 1 -> it runs unsplit
    # (13 ns, no overheads) after L: 15..28; s_max = 2 -> split, 15..30
    assert qos.simulate(blocks, [0, 1], [0, 0], qos.ELASTIC, uns, big, 1) == [15, 27]
    assert qos.simulate(blocks, [0, 1], [0, 0], qos.ELASTIC, uns, big, 2) == [15, 29]
    # a queued unsplit request is passed by a later split arrival like any other:
    # Q = [L (left 10), L' (unsplit 13)]; S at 2: 13*15 > 4 and 10*15 > 4 -> head;
    # S runs at L's first block boundary 5..7, L 7..17, L' 17..30
    assert qos.simulate(blocks, [0, 1, 2], [0, 0, 1], qos.ELASTIC, uns, big, 1) == [17, 29, 5]


def test_elastic_thresholds_zero_is_fifo_lindley_of_unsplit_models():
    # d_max = 0: splitting always off -> a FIFO single-server queue whose service
    # time is the unsplit T of each request: end_i = max(a_i, end_{i-1}) + T(m_i)
    arr, ty = wl.qos_requests(2, 300, 6_000_000, 3, seed=11)
    blocks = wl.random_blocks(3, seed=4, k_hi=5, lo=500_000, hi=4_000_000)
    uns = [sum(b) - 300_000 for b in blocks]
    for r in range(2):
        a = [int(x) for x in arr[r]]
        t = [int(x) for x in ty[r]]
        for d, s in ((0, 1 << 30), (1 << 30, 0)):
            got = qos.simulate(blocks, a, t, qos.ELASTIC, uns, d, s)
            end = 0
            for i in range(len(a)):
                end = max(a[i], end) + uns[t[i]]
                assert got[i] == end - a[i]


def test_elastic_infinite_thresholds_is_algorithm1():
    arr, ty = wl.qos_requests(2, 200, 8_000_000, 4, seed=12)
    blocks = wl.random_blocks(4, seed=5, k_hi=5, lo=500_000, hi=6_000_000)
    uns = [sum(b) for b in blocks]
    for r in range(2):
        a = [int(x) for x in arr[r]]
        t = [int(x) for x in ty[r]]
        assert qos.simulate(blocks, a, t, qos.ELASTIC, uns, 1 << 30, 1 << 30) == qos.simulate(blocks, a, t, qos.ALG1)


def test_stats_against_an_isolated_reference():
    # §5.2 (P@33300-33700) measures response ratios against the isolated execution time; with
    # ref = the unsplit T per type the same latencies give, by hand: RR = 17/13 and 6/2 = 3;
    # at alpha = 2 only the second violates (6000 > 4000, 17000 <= 26000)
    viol, rs, rq = qos.stats([[5, 5, 5], [2]], [0, 1], [17, 6], [1000, 2000, 3000], ref=[13, 2])
    assert viol == [2, 1, 0]
    assert rs == 17 / 13 + 3.0 and rq == (17 / 13) ** 2 + 9.0
