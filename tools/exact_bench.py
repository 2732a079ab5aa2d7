"""Time split_exhaustive (f1) on a synthetic chain: splits/s with CUDA events
(split_last_run_stats) and wall clock.  Tuning aid."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402

if __name__ == "__main__":
    torch.cuda.set_device(0)
    for n in [int(a) for a in sys.argv[1:]] or [29, 33, 37]:
        lat, ovh = wl.random_chain(n, 3, ovh_hi=100_000)
        with S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=min(n, 32)) as h:
            h.exhaustive()
            t0 = time.perf_counter()
            r = h.exhaustive()
            wall = time.perf_counter() - t0
            st = h.last_run_stats()
        print(f"n={n:2d}  2^{n-1} splits  {st['ms_total']:9.3f} ms device  {wall*1e3:9.3f} ms wall  "
              f"{(2 ** (n - 1)) / (st['ms_total'] * 1e-3) / 1e9:8.1f} G splits/s  best k={r['k']} f={r['fitness']:.6f}")
