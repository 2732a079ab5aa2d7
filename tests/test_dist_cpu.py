"""World-size-2 gloo tests of the multi-process host logic (CPU only)."""
import os
import socket

import pytest
import torch.multiprocessing as mp

from paper_conf_icpp_luoyww0023_b200 import dist as D


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        uid = D.broadcast_bytes(bytes(range(128)) if rank == 0 else None)
        lay = D.island_layout(rank, world, 2)
        lo, hi = D.shard_range(1001, rank, world)
        t, c, e = D.reduce_max_sum(10.0 + rank, 100.0 * (rank + 1), 1.0)
        q.put((rank, uid, lay, (lo, hi), (t, c, e)))
    finally:
        dist.destroy_process_group()


def test_two_rank_gloo_plumbing():
    world, port = 2, _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, uid0, lay0, sh0, red0), (r1, uid1, lay1, sh1, red1) = res
    assert uid0 == uid1 == bytes(range(128))
    assert lay0 == {"island_id": 0, "n_islands": 4, "islands_per_device": 2}
    assert lay1 == {"island_id": 2, "n_islands": 4, "islands_per_device": 2}
    assert sh0 == (0, 501) and sh1 == (501, 1001)
    assert red0 == red1 == (11.0, 300.0, 2.0)


@pytest.mark.parametrize("n,world", [(0, 3), (7, 3), (1 << 20, 8), (5, 8)])
def test_shard_range_partitions(n, world):
    got = [D.shard_range(n, r, world) for r in range(world)]
    assert got[0][0] == 0 and got[-1][1] == n
    for (a, b), (c, d) in zip(got, got[1:]):
        assert b == c and b >= a
    assert max(b - a for a, b in got) - min(b - a for a, b in got) <= 1


def test_island_layout_rejects():
    with pytest.raises(ValueError):
        D.island_layout(2, 2)
