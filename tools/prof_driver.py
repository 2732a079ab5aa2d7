"""Minimal drivers for ncu captures (one GPU): `eval` runs split_eval_batch on C5,
`ga` runs split_ga_run on C2, `qos` the f2 simulator.  Not a benchmark (numbers under ncu are not bench values)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402


def main(what: str, reps: int = 3, gens: int = 500):
    torch.cuda.set_device(0)
    st = torch.cuda.current_stream()
    if what == "eval":
        lat, ovh = wl.chain("synthetic_1024")
        n_cand = 1 << 24
        h = S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=32, stream=st)
        bits = torch.from_numpy(wl.uniform_k_population_fast(len(lat), n_cand, seed=20230807).view(np.int64)).cuda()
        out = torch.empty(n_cand, dtype=torch.float64, device="cuda")
        for _ in range(reps):
            h.eval_batch(bits, n_cand, out)
        torch.cuda.synchronize()
    elif what in ("qos", "qos_el"):
        blocks = [[3_575_000, 3_031_000, 3_231_000, 3_191_000], [4_005_000, 4_052_000, 3_984_000, 4_040_000],
                  [8_984_000, 8_747_000, 8_865_000, 8_990_000], [22_314_000, 21_125_000, 18_922_000, 19_467_000],
                  [6_124_000, 6_154_000, 6_078_000, 6_139_000]]
        arr, typ = wl.qos_requests(65536, 1000, 110_000_000, 5, seed=2023)
        da = torch.from_numpy(np.ascontiguousarray(arr.T)).cuda()
        dt = torch.from_numpy(np.ascontiguousarray(typ.T)).cuda()
        kw = {}
        if what == "qos_el":     # f4 elastic (R23), the bench's thresholds
            kw = dict(unsplit=[sum(b) - 300_000 for b in blocks], d_max=3, s_max=2)
        for _ in range(reps):
            S.split_qos_simulate(blocks, da, dt, [1000 * a for a in range(2, 21)], 2 if kw else 1, **kw)
        torch.cuda.synchronize()
        return
    elif what in ("ga_big", "ga_1m"):
        lat, ovh = wl.chain("bert_base")
        h = S.SplitGA(lat, ovh, pop_size=(1 << 22) if what == "ga_big" else (1 << 20), n_elite=1024, k_min=2, k_max=32,
                      stream=st)
        for i in range(reps):
            h.run(gens, i)
    else:
        lat, ovh = wl.chain("resnet50_175")
        h = S.SplitGA(lat, ovh, pop_size=65536, n_elite=1024, k_min=2, k_max=32, stream=st)
        for i in range(reps):
            r = h.run(gens, i)
        print(r["fitness"], h.last_run_stats())
    h.close()


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 3, int(sys.argv[3]) if len(sys.argv) > 3 else 500)
