"""Steady-state GA generation time: run(G) for two G and difference the loop times, so the
initial generations (where crossover children still need repair) drop out.  Probe only."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S, workloads as wl  # noqa: E402

torch.cuda.set_device(0)
cases = [("resnet50_175", 65536, (100, 500)), ("bert_base", 1 << 20, (20, 220)), ("bert_base", 1 << 22, (20, 120))]
for chain, N, (g0, g1) in cases:
    lat, ovh = wl.chain(chain)
    h = S.SplitGA(lat, ovh, pop_size=N, n_elite=1024, k_min=2, k_max=32, stream=torch.cuda.current_stream())
    t = {}
    for G in (g0, g1, g0, g1):
        h.run(G, 5)
        t.setdefault(G, []).append(h.last_run_stats()["ms_loop"])
    a, b = min(t[g0]), min(t[g1])
    print(f"{chain} N={N}: G={g0} {a:.3f} ms, G={g1} {b:.3f} ms, steady {1000 * (b - a) / (g1 - g0):.1f} us/gen, "
          f"first {g0}: {1000 * a / g0:.1f} us/gen", flush=True)
    h.close()
