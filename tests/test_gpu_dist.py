"""Island model across processes (north_star: one island per GPU, top-K migrants
all-gathered over NCCL every M generations): G ranks, each running one island
through split_ga_run with a split_comm_init communicator, must reproduce the
oracle's serial islands bit for bit -- every island's population and the
global best -- the SURVEY §4 anchor "islands on G GPUs == batched on one GPU ==
oracle".  Needs at least two visible GPUs (skipped otherwise; the single-GPU
forms of the same check are in test_gpu_ga.py)."""
import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_icpp_luoyww0023_b200 import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

KW = dict(pop_size=512, n_elite=16, k_min=2, k_max=32, migration_interval=3, n_migrants=8)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _rank_main(rank, world, port, G, seed, out_dir):
    import torch.distributed as dist

    from paper_conf_icpp_luoyww0023_b200 import dist as D
    from paper_conf_icpp_luoyww0023_b200 import split as S
    torch.cuda.set_device(rank)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    uid = D.broadcast_bytes(S.split_comm_unique_id() if rank == 0 else None)
    comm = S.split_comm_init(uid, rank, world, rank)
    lat, ovh = wl.chain("resnet50_175")
    with S.SplitGA(lat, ovh, device=rank, comm=comm, **KW, **D.island_layout(rank, world, 1)) as h:
        r = h.run(G, seed)
        bits, fit = h.population(0)
    S.split_comm_destroy(comm)
    np.savez(os.path.join(out_dir, f"rank{rank}.npz"), bits=bits, fit=fit, best_bits=r["bits"],
             best_f=r["fitness"], gen_found=r["generation_found"], gens=r["generations_run"],
             evals=r["evaluations"])
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_islands_across_ranks_match_oracle(world, tmp_path):
    if not torch.cuda.is_available() or torch.cuda.device_count() < world:
        pytest.skip(f"needs {world} GPUs")
    import torch.multiprocessing as mp
    G, seed = 11, 2024
    mp.spawn(_rank_main, args=(world, _free_port(), G, seed, str(tmp_path)), nprocs=world, join=True)
    lat, ovh = wl.chain("resnet50_175")
    o = oracle.ga_run(lat, ovh, G, seed, n_islands=world, want_population=True, **KW)
    for rank in range(world):
        d = np.load(os.path.join(tmp_path, f"rank{rank}.npz"))
        assert np.array_equal(d["bits"], o["population"][rank]), f"island {rank} rows"
        assert np.array_equal(d["fit"].view(np.uint64), o["fitness_all"][rank].view(np.uint64))
        # every rank reports the same global best (R19), the oracle's
        assert float(d["best_f"]) == o["fitness"] and np.array_equal(d["best_bits"], o["bits"])
        assert int(d["gen_found"]) == o["generation_found"] and int(d["gens"]) == o["generations_run"]
