"""GPU parity of the f2 QoS simulator (split_qos_simulate, R20)
against oracle/qos.py (literal Algorithm 1 in exact rationals, or FIFO):
end-to-end latency of every request, violation counts per alpha and both
response-ratio sums, bit for bit.  Small cases compare every replica; the
bench-sized case (Table 2's 1000 requests, lambda = 110 ms, 8192 replicas)
compares sampled replicas plus properties that hold at any size."""
import numpy as np
import pytest

from oracle import qos as Q
from paper_conf_icpp_luoyww0023_b200 import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ALPHAS = [1000 * a for a in range(2, 21)] + [1500]


@pytest.fixture(scope="module")
def S():
    if not torch.cuda.is_available():
        pytest.fail("CUDA not available on a GPU test run")
    from paper_conf_icpp_luoyww0023_b200 import split
    return split


def _run(S, blocks, arr, ty, policy, alphas=ALPHAS):
    # replica-major in the tests, request-major at the ABI
    a = torch.from_numpy(np.ascontiguousarray(arr.T)).cuda()
    t = torch.from_numpy(np.ascontiguousarray(ty.T)).cuda()
    te, viol, rr = S.split_qos_simulate(blocks, a, t, alphas, policy)
    torch.cuda.synchronize()
    return np.ascontiguousarray(te.cpu().numpy().T), viol.cpu().numpy().view(np.uint32), rr.cpu().numpy()


def _check_replica(blocks, arr, ty, policy, te, viol, rr, alphas=ALPHAS):
    a = [int(x) for x in arr]
    t = [int(x) for x in ty]
    want = Q.simulate(blocks, a, t, policy)
    assert [int(x) for x in te] == want
    v, rs, rq = Q.stats(blocks, t, want, alphas)
    assert [int(x) for x in viol[:len(alphas)]] == v
    assert rr[0] == rs and rr[1] == rq          # bit-identical sums


@pytest.mark.parametrize("policy", [Q.FIFO, Q.ALG1])
@pytest.mark.parametrize("seed", [1, 42, 20230807])
def test_small_cases_all_replicas(S, policy, seed):
    blocks = wl.random_blocks(5, seed=seed, k_hi=6, lo=300_000, hi=9_000_000)
    arr, ty = wl.qos_requests(37, 150, 40_000_000, 5, seed=seed)   # ragged: 37 replicas (one partial CTA)
    te, viol, rr = _run(S, blocks, arr, ty, policy)
    for r in range(arr.shape[0]):
        _check_replica(blocks, arr[r], ty[r], policy, te[r], viol[r], rr[r])


def test_ties_and_degenerate_inputs(S):
    # simultaneous arrivals, arrival exactly at a block end, one-block models, one request
    blocks = [[5, 5, 5], [2], [7]]
    arr = np.array([[0, 0, 5, 5, 10, 17, 17, 30]], dtype=np.int64)
    ty = np.array([[0, 1, 1, 2, 0, 1, 1, 2]], dtype=np.int32)
    for pol in (Q.FIFO, Q.ALG1):
        te, viol, rr = _run(S, blocks, arr, ty, pol)
        _check_replica(blocks, arr[0], ty[0], pol, te[0], viol[0], rr[0])
    te, viol, rr = _run(S, [[5, 5, 5], [2]], np.array([[0, 1]], dtype=np.int64), np.array([[0, 1]], dtype=np.int32),
                        Q.ALG1, [1000, 2000, 3000])
    assert te[0].tolist() == [17, 6]          # the worked example of tests/test_oracle_qos.py
    assert viol[0].tolist() == [2, 1, 0]
    te, _, _ = _run(S, [[4]], np.array([[3]], dtype=np.int64), np.array([[0]], dtype=np.int32), Q.ALG1)
    assert te.tolist() == [[4]]


def test_table2_sized_run_sampled(S):
    # Table 2's heaviest scenario (lambda = 110 ms), 1000 requests, five models whose
    # blocks come from 4-way splits of the paper-five chains' totals
    tot = [10_800_000, 13_200_000, 28_350_000, 67_500_000, 20_400_000]
    rng = np.random.default_rng(11)
    blocks = []
    for T in tot:
        w = rng.uniform(0.8, 1.2, size=4)
        b = np.floor(T * w / w.sum()).astype(np.int64)
        blocks.append([int(x) for x in b])
    arr, ty = wl.qos_requests(8192, 1000, 110_000_000, 5, seed=7)
    for pol in (Q.FIFO, Q.ALG1):
        te, viol, rr = _run(S, blocks, arr, ty, pol)
        ext = np.array([sum(b) for b in blocks], dtype=np.int64)
        assert (te >= ext[ty]).all()                                # never faster than isolated
        assert (np.diff(viol[:, :19].astype(np.int64), axis=1) <= 0).all()   # monotone in alpha
        for r in (0, 4095, 8191):
            _check_replica(blocks, arr[r], ty[r], pol, te[r], viol[r], rr[r])


def test_error_paths(S):
    blocks = [[5]]
    a = torch.tensor([[5], [3]], dtype=torch.int64, device="cuda")        # arrivals out of order
    t = torch.zeros((2, 1), dtype=torch.int32, device="cuda")
    with pytest.raises(S.SplitError) as e:
        S.split_qos_simulate(blocks, a, t, [2000], 1)
    assert e.value.code == S.SPLIT_E_RANGE
    a = torch.zeros((200, 1), dtype=torch.int64, device="cuda")           # 200 simultaneous: > 160 pending
    t = torch.zeros((200, 1), dtype=torch.int32, device="cuda")
    with pytest.raises(S.SplitError) as e:
        S.split_qos_simulate(blocks, a, t, [2000], 0)
    assert e.value.code == S.SPLIT_E_RANGE
    a = torch.zeros((40, 1), dtype=torch.int64, device="cuda")
    t = torch.zeros((40, 1), dtype=torch.int32, device="cuda")
    with pytest.raises(S.SplitError) as e:
        S.split_qos_simulate([[0]], a, t, [2000], 0)                        # zero-length block
    assert e.value.code == S.SPLIT_E_RANGE


# ---- f4 elastic splitting (split_qos_simulate_elastic, R23) ----

BIG = (1 << 32) - 1


def _run_el(S, blocks, uns, d, s, arr, ty, alphas=ALPHAS, ref=None):
    a = torch.from_numpy(np.ascontiguousarray(arr.T)).cuda()
    t = torch.from_numpy(np.ascontiguousarray(ty.T)).cuda()
    te, viol, rr = S.split_qos_simulate(blocks, a, t, alphas, 2, unsplit=uns, d_max=d, s_max=s, ref=ref)
    torch.cuda.synchronize()
    return np.ascontiguousarray(te.cpu().numpy().T), viol.cpu().numpy().view(np.uint32), rr.cpu().numpy()


def _check_el(blocks, uns, d, s, arr, ty, te, viol, rr, alphas=ALPHAS, ref=None):
    a = [int(x) for x in arr]
    t = [int(x) for x in ty]
    want = Q.simulate(blocks, a, t, Q.ELASTIC, uns, d, s)
    assert [int(x) for x in te] == want
    v, rs, rq = Q.stats(blocks, t, want, alphas, ref)
    assert [int(x) for x in viol[:len(alphas)]] == v
    assert rr[0] == rs and rr[1] == rq


@pytest.mark.parametrize("d,s", [(0, BIG), (2, BIG), (BIG, 1), (3, 2), (BIG, BIG)])
@pytest.mark.parametrize("seed", [3, 2023])
def test_elastic_small_cases_all_replicas(S, d, s, seed):
    blocks = wl.random_blocks(5, seed=seed, k_hi=6, lo=300_000, hi=9_000_000)
    uns = [max(1, sum(b) - 150_000 * (len(b) - 1)) for b in blocks]     # no cut overheads
    arr, ty = wl.qos_requests(37, 150, 30_000_000, 5, seed=seed)
    te, viol, rr = _run_el(S, blocks, uns, d, s, arr, ty)
    for r in range(arr.shape[0]):
        _check_el(blocks, uns, d, s, arr[r], ty[r], te[r], viol[r], rr[r])
    if d == BIG and s == BIG:                 # no suspension: exactly policy 1
        te1, _, _ = _run(S, blocks, arr, ty, Q.ALG1)
        assert (te1 == te).all()


@pytest.mark.parametrize("d,s", [(2, BIG), (3, 2)])
def test_elastic_isolated_reference_all_replicas(S, d, s):
    # violations and RR against the isolated unsplit T (§5.2, P@33300-33700) instead of the split Ext:
    # the same schedule, a different denominator; a request served unsplit then has RR >= 1
    blocks = wl.random_blocks(5, seed=7, k_hi=6, lo=300_000, hi=9_000_000)
    uns = [max(1, sum(b) - 150_000 * (len(b) - 1)) for b in blocks]
    arr, ty = wl.qos_requests(37, 150, 30_000_000, 5, seed=7)
    te, viol, rr = _run_el(S, blocks, uns, d, s, arr, ty, ref=uns)
    te0, _, _ = _run_el(S, blocks, uns, d, s, arr, ty)
    assert (te == te0).all()
    for r in range(arr.shape[0]):
        _check_el(blocks, uns, d, s, arr[r], ty[r], te[r], viol[r], rr[r], ref=uns)
    assert (rr[:, 0] >= 150 - 1e-9).all()       # every t_ete >= the isolated T of its type


def test_elastic_worked_examples(S):
    blocks, uns = [[5, 5, 5], [2]], [13, 2]
    one = lambda a, t, d, s: _run_el(S, blocks, uns, d, s, np.array([a], dtype=np.int64),
                                     np.array([t], dtype=np.int32), [2000])[0][0].tolist()
    assert one([0, 1], [0, 1], 1, BIG) == [15, 16]      # tests/test_oracle_qos.py, by hand
    assert one([0, 1], [0, 1], 2, BIG) == [17, 6]
    assert one([0, 1], [0, 0], BIG, 1) == [15, 27]
    assert one([0, 1, 2], [0, 0, 1], BIG, 1) == [17, 29, 5]


def test_elastic_table2_sized_run_sampled(S):
    tot = [10_800_000, 13_200_000, 28_350_000, 67_500_000, 20_400_000]
    rng = np.random.default_rng(13)
    blocks = []
    for T in tot:
        w = rng.uniform(0.8, 1.2, size=4)
        blocks.append([int(x) for x in np.floor(T * w / w.sum()).astype(np.int64)])
    uns = [sum(b) - 3 * 400_000 for b in blocks]
    arr, ty = wl.qos_requests(8192, 1000, 110_000_000, 5, seed=8)
    te, viol, rr = _run_el(S, blocks, uns, 2, 3, arr, ty)
    assert (te >= np.array(uns, dtype=np.int64)[ty]).all()
    for r in (0, 4095, 8191):
        _check_el(blocks, uns, 2, 3, arr[r], ty[r], te[r], viol[r], rr[r])


def test_elastic_error_paths(S):
    a = torch.zeros((2, 1), dtype=torch.int64, device="cuda")
    t = torch.zeros((2, 1), dtype=torch.int32, device="cuda")
    with pytest.raises(S.SplitError) as e:
        S.split_qos_simulate([[5]], a, t, [2000], 2, unsplit=[0], d_max=1, s_max=1)   # unsplit time 0
    assert e.value.code == S.SPLIT_E_RANGE
    with pytest.raises(S.SplitError) as e:
        S.split_qos_simulate([[5]], a, t, [2000], 3)                                   # no such policy
    assert e.value.code == S.SPLIT_E_INVAL


@pytest.mark.parametrize("pol", [Q.FIFO, Q.ALG1, Q.ELASTIC])
def test_overloaded_queue_rerun(S, pol):
    """More than 32 pending requests in some replicas (bursts of simultaneous arrivals, a load
    Table 2 never reaches): the library re-runs the batch with the 160-entry queue; every replica
    still matches the literal oracle (round 1 returned SPLIT_E_RANGE here)."""
    blocks = wl.random_blocks(3, seed=11, k_hi=4, lo=1_000_000, hi=5_000_000)
    rng = np.random.default_rng(11)
    n_rep, n_req = 8, 120
    arr = np.sort(rng.integers(0, 40_000_000, size=(n_rep, n_req)), axis=1).astype(np.int64)
    arr[:, :60] = 1000                                    # a burst of 60 simultaneous arrivals
    arr = np.sort(arr, axis=1)
    ty = rng.integers(0, 3, size=(n_rep, n_req)).astype(np.int32)
    uns = [max(1, sum(b) - 50_000) for b in blocks]
    kw = dict(unsplit=uns, d_max=40, s_max=30) if pol == Q.ELASTIC else {}
    te, viol, rr = S.split_qos_simulate(blocks, torch.from_numpy(np.ascontiguousarray(arr.T)).cuda(),
                                        torch.from_numpy(np.ascontiguousarray(ty.T)).cuda(), ALPHAS, pol, **kw)
    torch.cuda.synchronize()
    te = np.ascontiguousarray(te.cpu().numpy().T)
    for r in range(n_rep):
        args = (uns, 40, 30) if pol == Q.ELASTIC else ()
        assert [int(x) for x in te[r]] == Q.simulate(blocks, arr[r].tolist(), ty[r].tolist(), pol, *args)
