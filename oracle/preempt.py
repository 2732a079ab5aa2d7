"""Literal Algorithm 1 (greedy preemption, §3.4 / Alg. 1, P@27209-28515).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Every response ratio is an
exact ``fractions.Fraction`` (Eq. 3, P@24997-25459), so the comparison on line
13 is decided without rounding.  It does NOT use the closed form the library
implements (DESIGN.md §3 R12); the tests check that the two agree.

Readings of the garbled pseudo-code (DESIGN.md §3 R12):
  * line 4 sums Ext_left (the remaining work of the requests ahead), not Ext;
  * line 5 scans from the tail (the request right ahead of t_new) to the head,
    because l_waiting shrinks by Ext_left(t_i) on each step (line 9);
  * line 6 / 14 "return T" / "T.insert(t_i, t_new)" leave t_new right behind t_i;
  * line 11 adds the work t_new puts in front of t_i (Ext_left(t_new)) — the
    printed "+Ext_left(t_i)" would make t_i wait behind itself;
  * line 19 "T.end" is the head of the queue (highest priority, P@26642-26663);
  * clock() - Start(t) is the time t has waited since it arrived (Eq. 3).
Queue convention: queue[0] is the head (runs next); the result is the index at
which t_new is inserted (0 = head, n = tail).
"""
from __future__ import annotations

from dataclasses import dataclass
from fractions import Fraction


@dataclass(frozen=True)
class Request:
    type_id: int
    arrival_ns: int
    ext_ns: int        # Ext(t): execution time of the request
    ext_left_ns: int   # Ext_left(t): remaining execution time


def response_ratio(now_ns: int, alpha: float, l_waiting: int, t: Request) -> Fraction:
    """Function ResponseRatio, lines 1-3."""
    l_waited = now_ns - t.arrival_ns                       # line 1
    target = Fraction(alpha) * t.ext_ns                    # line 2
    return Fraction(l_waited + l_waiting + t.ext_left_ns) / target   # line 3


def preemption(now_ns: int, alpha: float, queue: list[Request], t_new: Request) -> int:
    """Function Preemption, lines 4-20; returns the insertion index of t_new."""
    n = len(queue)
    l_waiting = sum(t.ext_left_ns for t in queue)          # line 4
    for i in range(n - 1, -1, -1):                         # line 5 (tail -> head)
        t_i = queue[i]
        if t_new.type_id == t_i.type_id:                   # line 6
            return i + 1
        rr_new_back = response_ratio(now_ns, alpha, l_waiting, t_new)              # line 8
        l_waiting -= t_i.ext_left_ns                                                # line 9
        rr_new_front = response_ratio(now_ns, alpha, l_waiting, t_new)             # line 10
        rr_i_back = response_ratio(now_ns, alpha, l_waiting + t_new.ext_left_ns, t_i)  # line 11
        rr_i_front = response_ratio(now_ns, alpha, l_waiting, t_i)                 # line 12
        if rr_new_front - rr_new_back >= rr_i_front - rr_i_back:                   # line 13
            return i + 1                                                            # line 14-15
    return 0                                                                        # line 19


def sum_rr(now_ns: int, alpha: float, order: list[Request]) -> Fraction:
    """Sum of Eq. 3 response ratios of a queue executed in the given order."""
    total = Fraction(0)
    ahead = 0
    for t in order:
        total += response_ratio(now_ns, alpha, ahead, t)
        ahead += t.ext_left_ns
    return total
