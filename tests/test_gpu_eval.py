"""GPU parity of the device RNG, dexp and split_eval_batch (a2) against the CPU
oracle — bit-exact (fitness is exact integer statistics + a pinned FP64 tail,
DESIGN.md R5'/R5'').  All calls go through the C ABI."""
import math

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


def _bits_equal(a, b):
    return np.array_equal(np.asarray(a, np.float64).view(np.uint64), np.asarray(b, np.float64).view(np.uint64))


def test_device_philox_matches_oracle(S):
    rng = np.random.default_rng(0)
    ck = rng.integers(0, 2 ** 32, size=(5000, 6), dtype=np.uint64).astype(np.uint32)
    ck[0] = 0
    ck[1] = 0xFFFFFFFF
    ck[2] = [0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344, 0xa4093822, 0x299f31d0]
    got = S.split_selftest_philox(ck)
    assert tuple(got[0]) == (0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8)
    assert tuple(got[2]) == (0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1)
    for i in range(0, 5000, 7):
        assert tuple(got[i]) == oracle.philox(ck[i, :4], ck[i, 4:])


def test_device_dexp_bit_exact(S):
    rng = np.random.default_rng(1)
    z = np.concatenate([rng.uniform(-1, 3, 200000), rng.uniform(-1, 709.7, 20000),
                        [-1.0, 0.0, 0.5, 1.0, 709.0, 709.78, 710.0, 711.0]])
    got = S.split_selftest_dexp(z)
    ref = np.array([oracle.dexp(float(v)) for v in z])
    assert _bits_equal(got, ref)


def _eval_gpu(S, lat, ovh, bits, k_min, k_max):
    n = len(lat)
    h = S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=k_min, k_max=k_max)
    d = torch.from_numpy(np.ascontiguousarray(bits).view(np.int64)).cuda()
    out = h.eval_batch(d, bits.shape[0])
    torch.cuda.synchronize()
    h.close()
    return out.cpu().numpy()


@pytest.mark.parametrize("kind", ["profile", "const", "zero", "ties"])
def test_c1_exhaustive_eval(S, kind):
    lat, ovh = wl.c1_chain(overhead=kind)
    bits = np.arange(2048, dtype=np.uint64).reshape(-1, 1)
    got = _eval_gpu(S, lat, ovh, bits, 1, 12)
    ref = oracle.fitness_batch(lat, ovh, bits, 1, 12)
    assert _bits_equal(got, ref)
    # and with the GA's k range: k outside [2, 12] -> -inf
    got2 = _eval_gpu(S, lat, ovh, bits, 2, 12)
    assert got2[0] == -math.inf and _bits_equal(got2[1:], ref[1:])


@pytest.mark.parametrize("n", [2, 3, 12, 37, 64, 65, 66, 105, 128, 129, 175, 400,
                               961, 993, 1000, 1024, 1025, 2534])   # W = 16 (swizzled K1): every padding shape
def test_random_batches_and_edges(S, n):
    scale = max(1, n // 64)          # keep (k_max-1) * T'^2 < 2^63 with k_max = n (a0 guard)
    lat, ovh = wl.random_chain(n, 1000 + n, lo=0, hi=200_000 // scale, ovh_hi=30_000 // scale)
    lat[0] = max(lat[0], 1)
    W = wl.words(n)
    kmax = min(n, 40)
    pop = [wl.sparse_population(n, 3000, seed=n, k_lo=1, k_hi=kmax)]
    edges = np.zeros((6, W), dtype=np.uint64)
    edges[1] = np.uint64(0xFFFFFFFFFFFFFFFF)                 # all ones (k = n: out of range unless n <= 40)
    edges[2, 0] = np.uint64(1)                                # cut after op 0
    p = n - 2
    edges[3, p >> 6] |= np.uint64(1) << np.uint64(p & 63)    # cut before the last op
    edges[4] = edges[2] | edges[3]
    if (n - 1) % 64:
        edges[5, W - 1] = ~np.uint64((1 << ((n - 1) % 64)) - 1)  # padding bits only -> k = 1
    pop.append(edges)
    pop.append(wl.dense_population(n, 257, seed=n, with_padding=True))
    bits = np.concatenate(pop)
    for kmin, kmax_ in [(1, n), (2, kmax)]:
        got = _eval_gpu(S, lat, ovh, bits, kmin, kmax_)
        ref = oracle.fitness_batch(lat, ovh, bits, kmin, kmax_)
        assert _bits_equal(got, ref), (n, kmin, kmax_)


def test_empty_and_ragged_batches(S):
    lat, ovh = wl.chain("bert_base")
    h = S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=32)
    bits = wl.sparse_population(len(lat), 1000, seed=5)
    d = torch.from_numpy(bits.view(np.int64)).cuda()
    out = torch.full((1000,), 7.0, dtype=torch.float64, device="cuda")
    h.eval_batch(d, 0, out)                                   # no-op
    torch.cuda.synchronize()
    assert float(out[0]) == 7.0
    for m in (1, 31, 32, 33, 999):
        o = h.eval_batch(d, m)
        torch.cuda.synchronize()
        assert _bits_equal(o.cpu().numpy(), oracle.fitness_batch(lat, ovh, bits[:m], 2, 32))
    # misaligned device pointer
    with pytest.raises(S.SplitError) as ei:
        h.eval_batch(d.data_ptr() + 8, 10, out)
    assert ei.value.code == S.SPLIT_E_ALIGN
    h.close()


def test_eval_batch_host_path(S):
    lat, ovh = wl.chain("resnet50_175")
    bits = wl.sparse_population(len(lat), 20000, seed=9)
    h = S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=32)
    got = h.eval_batch_host(bits)
    h.close()
    assert _bits_equal(got, oracle.fitness_batch(lat, ovh, bits, 2, 32))


def test_c5_full_size_sampled(S):
    """C5 at the size bench.py times (n = 1024, N = 2^24): outputs sampled and
    recomputed one by one by the oracle."""
    lat, ovh = wl.chain("synthetic_1024")
    n = len(lat)
    N = 1 << 24
    bits = wl.uniform_k_population_fast(n, N, seed=20230807)
    h = S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=32)
    d = torch.from_numpy(bits.view(np.int64)).cuda()
    out = h.eval_batch(d, N).cpu().numpy()
    h.close()
    rng = np.random.default_rng(3)
    idx = np.concatenate([rng.integers(0, N, 4000), np.arange(64), np.arange(N - 64, N)])
    ref = oracle.fitness_batch(lat, ovh, bits[idx], 2, 32)
    assert _bits_equal(out[idx], ref)
    assert np.isfinite(out).mean() > 0.95
