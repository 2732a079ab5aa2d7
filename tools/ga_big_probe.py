import sys, os, time
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_luoyww0023_b200 import split as S, workloads as wl
torch.cuda.set_device(0)
lat, ovh = wl.chain("bert_base")
for N in (1 << 20, 1 << 22):
    h = S.SplitGA(lat, ovh, pop_size=N, n_elite=1024, k_min=2, k_max=32, stream=torch.cuda.current_stream())
    for G in (50, 200):
        r = h.run(G, 5)
        st = h.last_run_stats()
        print(N, G, "ms_loop", round(st["ms_loop"], 2), "per gen us", round(1000 * st["ms_loop"] / G, 1), "general", st["general_selects"], "fast", st["fast_selects"])
    h.close()
