"""Time split_eval_batch (K1) with CUDA events on the handle's stream over the
C5 population recipe and a few chain widths; prints G evals/s and algorithmic
GB/s per case.  Tuning aid (the bench line comes from bench.py)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402


def time_case(name, n_cand, reps=20, dense=False, k_max=32):
    lat, ovh = wl.chain(name)
    st = torch.cuda.current_stream()
    h = S.SplitGA(lat, ovh, pop_size=4, n_elite=0, k_min=2, k_max=k_max, stream=st)
    W = h.W
    if dense:
        rng = np.random.default_rng(7)
        pop = rng.integers(0, 2**63, size=(n_cand, W), dtype=np.int64)
    else:
        pop = wl.uniform_k_population_fast(len(lat), n_cand, seed=20230807).view(np.int64)
    bits = torch.from_numpy(pop).cuda()
    out = torch.empty(n_cand, dtype=torch.float64, device="cuda")
    for _ in range(3):
        h.eval_batch(bits, n_cand, out)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(reps):
        h.eval_batch(bits, n_cand, out)
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    ge = n_cand / ms / 1e6
    gbs = n_cand * (8 * W + 8) / ms / 1e6
    print(f"{name:16s} W={W:2d} N={n_cand:>9d} dense={int(dense)}  {ms:8.3f} ms  {ge:7.2f} G evals/s  {gbs:7.1f} GB/s")
    h.close()
    return ms


if __name__ == "__main__":
    torch.cuda.set_device(0)
    if len(sys.argv) > 1 and sys.argv[1] == "c5":
        time_case("synthetic_1024", 1 << 24)
        sys.exit(0)
    time_case("synthetic_1024", 1 << 24)
    time_case("synthetic_1024", 1 << 24, dense=True)
    time_case("bert_base", 1 << 24)
    time_case("resnet50_175", 1 << 24)
    time_case("vgg16", 1 << 24)
