"""Pins for the literal Algorithm 1 oracle (P@27209-28515, Eq. 3 P@24997-25459).

Algorithm 1 swaps t_new with its neighbour while that lowers the two requests'
summed response ratio (§3.4, P@26152-26824).  What the mathematics fixes:
  * the swap test does not depend on alpha or on how long anyone has waited
    (both cancel in line 13's differences);
  * on a queue of distinct-type requests already in Smith (WSPT) order of
    Ext_left*Ext, the greedy position minimises the total response ratio over
    every possible insertion position (exchange argument);
  * an empty queue admits t_new at the head; a same-type tail keeps FIFO.
"""
import random

import pytest

from oracle.preempt import Request, preemption, sum_rr


def _rand_req(rng, type_id=None, now=10_000_000):
    ext = rng.randint(1, 200_000)
    left = rng.randint(0, ext)
    return Request(type_id if type_id is not None else rng.randint(0, 5),
                   now - rng.randint(0, 5_000_000), ext, left)


def test_empty_queue_and_same_type_tail():
    rng = random.Random(0)
    new = _rand_req(rng, 1)
    assert preemption(0, 2.0, [], new) == 0
    q = [_rand_req(rng, 2) for _ in range(5)] + [_rand_req(rng, 1)]
    assert preemption(10_000_000, 4.0, q, new) == len(q)


def test_independent_of_alpha_and_waits():
    rng = random.Random(1)
    for _ in range(300):
        n = rng.randint(0, 12)
        q = [_rand_req(rng) for _ in range(n)]
        new = _rand_req(rng)
        ref = preemption(10_000_000, 2.0, q, new)
        for alpha in (3.0, 7.5, 20.0):
            assert preemption(10_000_000, alpha, q, new) == ref
        q2 = [Request(t.type_id, t.arrival_ns - rng.randint(0, 10 ** 6), t.ext_ns, t.ext_left_ns) for t in q]
        assert preemption(10_000_000, 2.0, q2, new) == ref


def test_greedy_optimal_on_wspt_queue():
    rng = random.Random(2)
    checked = 0
    for _ in range(400):
        n = rng.randint(0, 9)
        q = [_rand_req(rng, type_id=10 + i) for i in range(n)]
        q.sort(key=lambda t: t.ext_left_ns * t.ext_ns)
        new = _rand_req(rng, type_id=99)
        now = 10_000_000
        pos = preemption(now, 2.0, q, new)
        costs = [sum_rr(now, 2.0, q[:i] + [new] + q[i:]) for i in range(n + 1)]
        assert costs[pos] == min(costs)
        checked += 1
    assert checked == 400


def test_single_swap_decision_is_exact():
    # one request ahead, different type: pass it iff the swap lowers the RR sum
    rng = random.Random(3)
    for _ in range(500):
        a = _rand_req(rng, 1)
        new = _rand_req(rng, 2)
        now, alpha = 10_000_000, 5.0
        behind = sum_rr(now, alpha, [a, new])
        ahead = sum_rr(now, alpha, [new, a])
        pos = preemption(now, alpha, [a], new)
        assert pos == (0 if ahead < behind else 1)
