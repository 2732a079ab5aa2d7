"""f4 elastic splitting (R23): when does suspending splitting pay?

Sweeps the thresholds (d_max, s_max) of split_qos_simulate_elastic against
Algorithm 1 (always split) and FIFO over split models whose cut overhead is a
fraction rho of the model's latency T per cut (4 equal blocks, the block after
a cut pays the overhead, R3), at two Poisson request rates (Table 2's
lambda = 110 ms and a denser 70 ms).  The models' T are the paper-five chain
totals (yolov2, googlenet, resnet50, vgg19, gpt2 as in bench.py).  Prints one
JSON object; the GPU run's output is kept in profiles/r02_elastic_sweep.json.
Violation rates and mean response ratios are reported against two latency
references (advisor round 1): the split model's Ext (the simulator's default,
R20/R23) and the isolated unsplit T that §5.2 (P@33300-33700) measures against
-- computed here from the returned per-request latencies.  Overloaded runs (a
replica with > 32 pending requests) are re-run by the library with its large
queue.  A measurement of the method's behaviour on synthetic inputs, not a
benchmark.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_luoyww0023_b200 import split as S  # noqa: E402
from paper_conf_icpp_luoyww0023_b200 import workloads as wl  # noqa: E402

N_REP, N_REQ = 16384, 1000
BIG = (1 << 32) - 1
ALPHAS = [2000, 3000, 5000]


def main():
    T = [int(np.asarray(wl.chain(m)[0], dtype=np.int64).sum()) for m in ("yolov2", "googlenet", "resnet50_122", "vgg19", "gpt2")]
    out = {"models_T_ms": [t / 1e6 for t in T], "n_rep": N_REP, "n_req": N_REQ, "runs": []}
    for lam_ms in (110, 70):
        arr, ty = wl.qos_requests(N_REP, N_REQ, lam_ms * 1_000_000, len(T), seed=31)
        da = torch.from_numpy(np.ascontiguousarray(arr.T)).cuda()
        dt = torch.from_numpy(np.ascontiguousarray(ty.T)).cuda()
        for rho in (0.0, 0.05, 0.15, 0.30):
            blocks = []
            for t in T:
                q = t // 4
                blocks.append([q] + [q + int(rho * t)] * 3)
            runs = [("algorithm1", 1, {}), ("fifo", 0, {})]
            for d in (1, 2, 3, 5, BIG):
                for s in (1, 2, BIG):
                    if d == BIG and s == BIG:
                        continue
                    runs.append((f"elastic d={'inf' if d == BIG else d} s={'inf' if s == BIG else s}", 2,
                                 dict(unsplit=T, d_max=d, s_max=s)))
            ext = np.array([sum(b) for b in blocks], dtype=np.float64)
            iso = np.array(T, dtype=np.float64)
            tyn = ty.T                                  # request-major, as te
            for name, pol, kw in runs:
                try:
                    te, viol, rr = S.split_qos_simulate(blocks, da, dt, ALPHAS, pol, **kw)
                except S.SplitError as e:          # > 160 pending even in the large queue
                    out["runs"].append({"lambda_ms": lam_ms, "rho": rho, "policy": name, "error": str(e)})
                    continue
                torch.cuda.synchronize()
                ten = te.cpu().numpy().astype(np.float64)
                rec = {"lambda_ms": lam_ms, "rho": rho, "policy": name}
                for ref_name, ref in (("split_ext", ext), ("isolated_T", iso)):
                    rrv = ten / ref[tyn]
                    rec[ref_name] = {"viol": {f"alpha={a // 1000}": round(float((rrv > a / 1000).mean()), 6)
                                              for a in ALPHAS},
                                     "rr_mean": round(float(rrv.mean()), 4)}
                out["runs"].append(rec)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
