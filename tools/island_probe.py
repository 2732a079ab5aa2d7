"""Island-loop overhead probe (tuning aid, one GPU): I batched islands of C2 size
(n = 175, N = 65,536 each) run 500 generations with migration every M
generations through a 1-rank NCCL communicator, against the same islands with
M = 0 (one RUN launch).  Prints gens/s and the cost of one sync point."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402


def run(I, M, G=500, reps=3, comm=None):
    lat, ovh = wl.chain("resnet50_175")
    st = torch.cuda.current_stream()
    kw = dict(pop_size=65536, n_elite=1024, k_min=2, k_max=32, n_islands=I, islands_per_device=I,
              migration_interval=M, n_migrants=64 if M else 0)
    with S.SplitGA(lat, ovh, stream=st, comm=comm, **kw) as h:
        h.run(G, 1)
        ms = []
        for i in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            r = h.run(G, 2 + i)
            e1.record(st)
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
    ms = sorted(ms)[len(ms) // 2]
    return ms, r


if __name__ == "__main__":
    torch.cuda.set_device(0)
    uid = S.split_comm_unique_id()
    comm = S.split_comm_init(uid, 0, 1, 0)
    G = 500
    if len(sys.argv) == 3:                      # one configuration, one run (for ncu launch lists)
        t, _ = run(int(sys.argv[1]), int(sys.argv[2]), G, reps=1, comm=comm)
        print(f"I={sys.argv[1]} M={sys.argv[2]} {t:.2f} ms")
        S.split_comm_destroy(comm)
        sys.exit(0)
    for I in (1, 8):
        base, _ = run(I, 0, G, comm=None if I == 1 else comm)
        print(f"I={I} M=0   {base:8.2f} ms  {G / base * 1e3:9.0f} gens/s", flush=True)
        if I == 1:
            continue
        for M in (10, 50):
            t, r = run(I, M, G, comm=comm)
            syncs = G // M - (1 if G % M == 0 else 0)
            print(f"I={I} M={M:<3d} {t:8.2f} ms  {G / t * 1e3:9.0f} gens/s  ratio {base / t:.3f}  "
                  f"per sync point {(t - base) / max(syncs, 1) * 1e3:8.1f} us", flush=True)
    S.split_comm_destroy(comm)
