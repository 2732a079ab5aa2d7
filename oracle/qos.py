"""QoS simulator oracle — TEST INFRASTRUCTURE ONLY.

A literal, slow, event-by-event simulation of one edge executor serving
requests of several split models, with the queue order decided at every
arrival by the literal Algorithm 1 of oracle/preempt.py (exact rationals),
or by FIFO.  Follows the system PAPER.md describes: requests are queued and
preempted only between blocks (§3.4 P@24400-26700: "Preemption can only be
executed between neighbors"; the blocks are the split's, §3.3), the latency
target is alpha x Ext (fn. 3, P@29746-29870), a request violates it when its
response ratio t_ete / t_ext (Eq. 3, P@24997-25459) exceeds alpha (§5.2,
P@33300-33700), arrivals are Poisson (§5.1 Table 2, P@31725-32980).  The
pinned event semantics are DESIGN.md reading R20:

* one executor; a block, once started, runs to completion;
* the pending queue Q holds every request with blocks not yet started, head
  first; Ext_left of an entry = the sum of its blocks not yet started;
* at an arrival (time a) the request (Ext_left = Ext) is inserted at the index
  the policy returns; an arrival at the same instant as a block end is
  processed first;
* whenever the executor is idle and Q is non-empty (after an arrival or a
  block end) it starts the next block of Q's head; a request whose last block
  has started leaves Q; its end-to-end latency t_ete = end of its last block
  minus its arrival.

f4 elastic splitting (ELASTIC, reading R23; §3.3 P@22612-23675:
splitting "is temporarily disabled" under "particularly high request density"
and "temporarily suspended" when "an excessive number of requests of the same
type are present"; the paper gives no thresholds, so they are parameters):
a request of type m arriving when Q holds >= d_max entries, or >= s_max
entries of type m, runs unsplit -- one block of unsplit[m] -- and is appended
at the tail of Q (no preemption); otherwise it is split and placed by
Algorithm 1 as under ALG1.  An unsplit entry in Q has Ext_left = unsplit[m].

Statistics (request order i = 0..n-1): violations per alpha = #{i : 1000 t_ete
> alpha_milli Ext}; rr_sum = sum of RN(t_ete/Ext) added in order, rr_sq = sum of
RN(RR*RR) added in order (IEEE doubles, as the CUDA path adds them).
"""
from __future__ import annotations

from dataclasses import dataclass

from oracle.preempt import Request, preemption

FIFO, ALG1, ELASTIC = 0, 1, 2


@dataclass
class _Entry:
    req: int
    ext_left: int
    blk: int
    unsplit: bool = False


def simulate(blocks: list[list[int]], arrival: list[int], types: list[int], policy: int,
             unsplit: list[int] | None = None, d_max: int = 0, s_max: int = 0) -> list[int]:
    """Return t_ete (ns) of every request.  unsplit, d_max, s_max: ELASTIC only."""
    n = len(arrival)
    ext = [sum(b) for b in blocks]
    t_ete = [None] * n
    Q: list[_Entry] = []
    busy_until = None          # end of the running block (None: idle)
    running = None             # request whose block is running
    running_last = False       # that block is its last
    i = 0                      # next arrival
    done = 0

    def dispatch(now):
        nonlocal busy_until, running, running_last
        if busy_until is not None or not Q:
            return
        h = Q[0]
        b = unsplit[types[h.req]] if h.unsplit else blocks[types[h.req]][h.blk]
        busy_until = now + b
        running = h.req
        h.blk += 1
        h.ext_left -= b
        running_last = h.ext_left == 0
        if running_last:
            Q.pop(0)

    while done < n:
        if busy_until is not None and (i >= n or busy_until < arrival[i]):
            now = busy_until                           # block end
            if running_last:
                t_ete[running] = now - arrival[running]
                done += 1
            busy_until = None
            running = None
            dispatch(now)
        else:
            now = arrival[i]                           # arrival (first on ties)
            m = types[i]
            entry = _Entry(i, ext[m], 0)
            same = sum(1 for e in Q if types[e.req] == m)
            if policy == FIFO:
                pos = len(Q)
            elif policy == ELASTIC and (len(Q) >= d_max or same >= s_max):
                entry = _Entry(i, unsplit[m], 0, True)         # splitting suspended (R23)
                pos = len(Q)
            else:
                queue = [Request(types[e.req], arrival[e.req], ext[types[e.req]], e.ext_left) for e in Q]
                pos = preemption(now, 1.0, queue, Request(m, now, ext[m], ext[m]))
            Q.insert(pos, entry)
            i += 1
            dispatch(now)
    return t_ete


def stats(blocks: list[list[int]], types: list[int], t_ete: list[int], alpha_milli: list[int],
          ref: list[int] | None = None):
    """(violations per alpha, rr_sum, rr_sq) in request order.  The latency
    reference of type m is ref[m] when given (e.g. the isolated unsplit T of
    §5.2, P@33300-33700), else Ext(m) = the sum of its split blocks (R20)."""
    ext = [sum(b) for b in blocks] if ref is None else list(ref)
    viol = [0] * len(alpha_milli)
    rr_sum = 0.0
    rr_sq = 0.0
    for i, t in enumerate(t_ete):
        e = ext[types[i]]
        for j, a in enumerate(alpha_milli):
            if 1000 * t > a * e:
                viol[j] += 1
        rr = float(t) / float(e)
        rr_sum = rr_sum + rr
        rr_sq = rr_sq + rr * rr
    return viol, rr_sum, rr_sq
