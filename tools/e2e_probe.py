import time, sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_luoyww0023_b200 import split as S, workloads as wl
torch.cuda.set_device(0)
lat, ovh = wl.chain("resnet50_175")
st = torch.cuda.current_stream()
for i in range(6):
    t0 = time.perf_counter()
    h = S.SplitGA(lat, ovh, pop_size=65536, n_elite=1024, k_min=2, k_max=32, stream=st)
    t1 = time.perf_counter()
    r = h.run(500, i)
    t2 = time.perf_counter()
    h.close()
    t3 = time.perf_counter()
    print(f"create {1e3*(t1-t0):7.2f} ms  run {1e3*(t2-t1):7.2f} ms  destroy {1e3*(t3-t2):7.2f} ms")
