cat > /tmp/probe.py <<'PY'
import sys, os
sys.path.insert(0, sys.argv[1])
import torch
from paper_conf_icpp_luoyww0023_b200 import split as S, workloads as wl
torch.cuda.set_device(0)
lat, ovh = wl.chain("resnet50_175"); st = torch.cuda.current_stream()
h = S.SplitGA(lat, ovh, pop_size=65536, n_elite=1024, k_min=2, k_max=32, stream=st)
h.run(500, 1); ms = []
for i in range(7):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st); h.run(500, 2 + i); e1.record(st); torch.cuda.synchronize(); ms.append(e0.elapsed_time(e1))
print(sys.argv[1], f"{sorted(ms)[3]:.3f} ms")
PY
for i in 1 2; do python /tmp/probe.py $PWD; python /tmp/probe.py $PWD/ab_r01; done
