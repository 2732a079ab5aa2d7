"""Small invocations of every kernel for compute-sanitizer (memcheck / racecheck / synccheck):
the GA kernel (INIT, RUN with batched islands and migration, 3 generations), K1 on W = 16 with a
ragged tail (swizzled tensor-TMA path) and on W = 3, the exhaustive f1 kernels and the DP, the f2 /
f4 simulators.  Checks results against nothing -- the parity suite does that; this only drives the
kernels under the tool."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402

what = sys.argv[1] if len(sys.argv) > 1 else "all"
torch.cuda.set_device(0)
if what in ("all", "ga"):
    lat, ovh = wl.chain("resnet50_175")
    with S.SplitGA(lat, ovh, pop_size=512, n_elite=16, k_min=2, k_max=16, n_islands=4, islands_per_device=4,
                   migration_interval=1, n_migrants=8) as h:
        h.run(3, 1)
    with S.SplitGA(lat, ovh, pop_size=4096, n_elite=64, k_min=2, k_max=32) as h:
        h.run(3, 2)
if what in ("all", "eval"):
    for name, n in (("synthetic_1024", 3000), ("resnet50_175", 1001)):
        lat, ovh = wl.chain(name)
        with S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=32) as h:
            bits = torch.from_numpy(wl.sparse_population(len(lat), n, seed=3).view(np.int64)).cuda()
            h.eval_batch(bits, n)
            h.heatmap2() if name == "resnet50_175" else None
if what in ("all", "exact"):
    lat, ovh = wl.random_chain(17, 3, ovh_hi=100_000)
    with S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=16) as h:
        h.exhaustive(per_k=True)
        h.dp_min_s2(16)
if what in ("all", "qos"):
    blocks = wl.random_blocks(5, seed=3, k_hi=6, lo=300_000, hi=9_000_000)
    arr, ty = wl.qos_requests(96, 60, 30_000_000, 5, seed=3)
    a = torch.from_numpy(np.ascontiguousarray(arr.T)).cuda()
    t = torch.from_numpy(np.ascontiguousarray(ty.T)).cuda()
    S.split_qos_simulate(blocks, a, t, [2000, 5000], 1)
    uns = [max(1, sum(b) - 150_000 * (len(b) - 1)) for b in blocks]
    S.split_qos_simulate(blocks, a, t, [2000, 5000], 2, unsplit=uns, d_max=3, s_max=2)
torch.cuda.synchronize()
print("sanitize driver done:", what)
