"""C2 step timing (tuning aid): split_ga_run of 500 generations on the ResNet-50 chain, N = 65,536."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402

torch.cuda.set_device(0)
lat, ovh = wl.chain("resnet50_175")
st = torch.cuda.current_stream()
with S.SplitGA(lat, ovh, pop_size=65536, n_elite=1024, k_min=2, k_max=32, stream=st) as h:
    h.run(500, 1)
    ms = []
    for i in range(5):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        h.run(500, 2 + i)
        e1.record(st)
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
print(f"C2 500 generations: {sorted(ms)[2]:.3f} ms per step (median of 5)")
