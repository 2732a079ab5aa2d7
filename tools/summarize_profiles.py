"""Turn a GPU round's raw outputs (gpurun_out/) into the committed summaries in
profiles/: launch-time shares, ncu key metrics, DRAM traffic per launch.

usage: python tools/summarize_profiles.py <round-tag>
"""
import collections
import csv
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.environ.get("SPLIT_PROF_OUT") or os.path.join(ROOT, "profiles")   # gpurun_out/ on the GPU box
REPS = os.environ.get("SPLIT_NCU_DIR") or OUT                                # where the .ncu-rep files are
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "nsecond": 1e-3, "us": 1.0,
         "usecond": 1.0, "ms": 1e3, "msecond": 1e3}


def launches(tag):
    path = os.path.join(OUT, "launches.csv")
    rows = list(csv.reader(open(path)))
    hdr, agg = None, collections.defaultdict(lambda: [0, 0.0])
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        us = float(d["Metric Value"].replace(",", "")) * SCALE.get(d["Metric Unit"], 1.0)
        agg[d["Kernel Name"].split("(")[0]][0] += 1
        agg[d["Kernel Name"].split("(")[0]][1] += us
    tot = sum(v[1] for v in agg.values())
    lines = [f"# Launch list ({tag}): `ncu --metrics gpu__time_duration.sum --clock-control none` over "
             "`bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-ga-big --no-qos` (cold-cache, serialised: "
             "compare shares; includes the eval_batch and f1 sub-measurements)", "",
             "| kernel | launches | total us | share |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k}` | {v[0]} | {v[1]:.1f} | {100 * v[1] / tot:.1f}% |")
    # the headline step (one split_ga_run) only: its kernels' shares
    step = {k: v for k, v in agg.items() if "ga_kernel" in k or "eval_stats_kernel" in k}
    st = sum(v[1] for v in step.values()) or 1.0
    lines += ["", "GA step only (split_ga_run: INIT + RUN launches and the best-record statistics kernel):", "",
              "| kernel | launches | total us | share of step |", "|---|---|---|---|"]
    for k, v in sorted(step.items(), key=lambda x: -x[1][1]):
        lines.append(f"| `{k}` | {v[0]} | {v[1]:.1f} | {100 * v[1] / st:.1f}% |")
    shutil.copy(path, os.path.join(PROF, f"{tag}_launches.csv"))
    return "\n".join(lines) + "\n"


def ncu_raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(txt.splitlines()))
    hdr, units, vals = rows[0], rows[1], rows[2]
    out = {"kernel": vals[hdr.index("Kernel Name")]}
    for k in KEYS:
        if k in hdr:
            i = hdr.index(k)
            try:
                out[k] = float(vals[i].replace(",", "")) * (SCALE.get(units[i], 1.0) if "bytes" in k else 1.0)
            except ValueError:
                out[k] = vals[i]
            out[k + ".unit"] = units[i]
    return out


def main(tag):
    os.makedirs(PROF, exist_ok=True)
    md = [launches(tag)]
    traffic = {}
    for name, rep, per in (("ga_kernel", "prof_ga.ncu-rep", "launch (one RUN segment = 500 generations of C2)"),
                           ("eval_batch_kernel", "prof_eval.ncu-rep", "launch (C5, 2^24 candidates)"),
                           ("ga_kernel, 1M island", "prof_ga_1m.ncu-rep",
                            "launch (C4 island: bert_base n=400, N=1,048,576, 20 generations from generation 0)"),
                           ("ga_kernel, 4M island", "prof_ga_4m.ncu-rep",
                            "launch (HBM regime: bert_base, N=4,194,304, 20 generations from generation 0)"),
                           ("qos_kernel", "prof_qos.ncu-rep", "launch (f2: 65,536 replicas x 1000 requests)"),
                           ("qos_kernel, f4 elastic", "prof_qos_el.ncu-rep",
                            "launch (f4: the same workload, d_max = 3, s_max = 2)")):
        path = os.path.join(REPS, rep)
        if not os.path.exists(path):
            continue
        m = ncu_raw(path)
        dram = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        traffic[name] = dram
        md.append(f"\n# ncu --set full: {name} (per {per})\n")
        md.append("| metric | value |\n|---|---|")
        for k in ["kernel"] + KEYS:
            if k in m:
                v = m[k]
                u = m.get(k + ".unit", "")
                md.append(f"| {k} | {v:,.3f} {u if 'bytes' not in k else 'B'} |" if isinstance(v, float) else f"| {k} | {v} |")
        md.append(f"| dram bytes (read+write) per launch | {dram:,.0f} B |")
    with open(os.path.join(PROF, f"{tag}_ncu_summary.md"), "w") as f:
        f.write("\n".join(md) + "\n")
    with open(os.path.join(PROF, "ncu_traffic.json"), "w") as f:
        json.dump({"round": tag, "ga_kernel_per_launch": traffic.get("ga_kernel"),
                   "eval_batch_kernel_c5": traffic.get("eval_batch_kernel")}, f, indent=1)
    if os.path.exists(os.path.join(OUT, "bench_full.json")):
        shutil.copy(os.path.join(OUT, "bench_full.json"), os.path.join(PROF, f"{tag}_bench.json"))
    print("\n".join(md))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "r01")
