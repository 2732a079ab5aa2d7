"""Multi-process plumbing for the island model (one process per GPU).

Pure host logic over torch.distributed (NCCL on the GPU box, gloo in the CPU
tests): island layout, the NCCL unique-id broadcast for split_comm_init,
contiguous sharding of split_eval_batch candidates (no exchange: candidates
are independent), and the max-over-ranks / sum-over-ranks reductions the
benchmark reports.  No method arithmetic lives here.
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def env_rank_world() -> tuple[int, int, int]:
    """(rank, world, local_rank) from the torchrun environment (1-process defaults)."""
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def island_layout(rank: int, world: int, islands_per_device: int = 1) -> dict:
    """Global islands [rank*ipd, (rank+1)*ipd) of world*ipd (split_ga_params fields)."""
    if world < 1 or not 0 <= rank < world or islands_per_device < 1:
        raise ValueError("bad layout")
    return {"island_id": rank * islands_per_device, "n_islands": world * islands_per_device,
            "islands_per_device": islands_per_device}


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous candidate rows [lo, hi) of rank r (first n % world ranks get one more)."""
    base, extra = divmod(n, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


def broadcast_bytes(payload: bytes | None, src: int = 0) -> bytes:
    """Broadcast an opaque byte string (the 128-byte NCCL unique id) from `src`."""
    obj = [payload]
    dist.broadcast_object_list(obj, src=src)
    return obj[0]


def reduce_max_sum(t_ms: float, count: float, extra: float = 0.0, device=None) -> tuple[float, float, float]:
    """(max over ranks of t_ms, sum over ranks of count, sum of extra)."""
    dev = device if device is not None else torch.device("cpu")
    t = torch.tensor([t_ms], dtype=torch.float64, device=dev)
    c = torch.tensor([count, extra], dtype=torch.float64, device=dev)
    if dist.is_available() and dist.is_initialized() and dist.get_world_size() > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dist.all_reduce(c, op=dist.ReduceOp.SUM)
    return float(t[0]), float(c[0]), float(c[1])
