"""Per-phase timing of the GA kernel's generation loop (C2), from the
%globaltimer probes compiled in with SPLIT_TRACE_BUILD=1 (tuning only: the
product build has none).  Usage on a GPU box:
    SPLIT_TRACE_BUILD=1 python -m paper_conf_icpp_luoyww0023_b200.build --force
    SPLIT_TRACE=gpurun_out/trace.csv python tools/trace_ga.py run
and here:  python tools/trace_ga.py show gpurun_out/trace.csv"""
import csv
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def run():
    import torch
    from paper_conf_icpp_luoyww0023_b200 import split as S
    from paper_conf_icpp_luoyww0023_b200 import workloads as wl
    torch.cuda.set_device(0)
    lat, ovh = wl.chain("resnet50_175")
    h = S.SplitGA(lat, ovh, pop_size=65536, n_elite=1024, k_min=2, k_max=32, stream=torch.cuda.current_stream())
    for seed in range(3):
        r = h.run(500, seed)
    print(r["fitness"])
    h.close()


def show(path):
    rows = list(csv.DictReader(open(path)))
    rows = [r for r in rows if int(r["work_start"]) and int(r["work_sync"])]
    pairs = [("work_start", "b_tourn", "tournament (fitness gathers)"),
             ("b_tourn", "b_rows", "parent rows"),
             ("b_rows", "b_xover", "crossover"),
             ("b_xover", "b_repair", "mutate + repair"),
             ("b_repair", "b_eval", "fused eval"),
             ("b_eval", "b_cand", "store + candidate append"),
             ("b_cand", "b_rec", "record filter"),
             ("b_rec", "work_end", "snapshot + CTA sync"),
             ("work_end", "work_sync", "grid barrier (worker)"),
             ("lead_start", "lead_loaded", "leader: TMA loads"),
             ("lead_loaded", "lead_record", "leader: record"),
             ("lead_record", "lead_sort", "leader: gather + sort"),
             ("lead_sort", "lead_end", "leader: merge + copy"),
             ("lead_end", "lead_sync", "grid barrier (leader)")]
    for a, b, name in pairs:
        d = sorted(int(r[b]) - int(r[a]) for r in rows if int(r[a]) and int(r[b]))
        if d:
            print(f"{name:32s} median {d[len(d) // 2] / 1e3:7.2f} us   p90 {d[int(len(d) * 0.9)] / 1e3:7.2f} us")
    per = sorted(int(rows[i + 1]["work_sync"]) - int(rows[i]["work_sync"]) for i in range(len(rows) - 1))
    print(f"{'generation (worker sync to sync)':32s} median {per[len(per) // 2] / 1e3:7.2f} us")
    # generation by generation (the first ones of a run are the slow ones): sync-to-sync and the
    # leader's phases, to see where the early generations spend their time
    for i in range(min(len(rows) - 1, 24)):
        r, q = rows[i], rows[i + 1]
        ph = {name: (int(r[b]) - int(r[a])) / 1e3 for a, b, name in pairs if int(r[a]) and int(r[b])}
        lead = " ".join(f"{n.split(': ')[-1]} {v:.1f}" for n, v in ph.items() if n.startswith("leader"))
        work = " ".join(f"{n.split(' (')[0]} {v:.1f}" for n, v in ph.items() if not n.startswith("leader"))
        print(f"gen {i:2d}: {(int(q['work_sync']) - int(r['work_sync'])) / 1e3:6.2f} us | {lead} | {work}")


def arrivals(path):
    """Per-CTA arrival spread at the generation barrier (SPLIT_TRACE=<p> writes <p>.arrivals)."""
    rows = [list(map(int, ln.split(","))) for ln in open(path) if ln.strip()]
    for r in rows:
        t = [x for x in r[1:] if x]
        if not t:
            continue
        lo = min(t)
        d = sorted((x - lo, c) for c, x in enumerate(r[1:]) if x)
        lead = r[1] - lo
        print(f"gen {r[0]}: leader arrives +{lead / 1e3:.2f} us; workers median +{d[len(d) // 2][0] / 1e3:.2f}, "
              f"p90 +{d[int(len(d) * 0.9)][0] / 1e3:.2f}, last +{d[-1][0] / 1e3:.2f} us (CTA {d[-1][1]}); "
              f"slowest 5: {[c for _, c in d[-5:]]}")


if __name__ == "__main__":
    if sys.argv[1] == "run":
        run()
    elif sys.argv[1] == "arrivals":
        arrivals(sys.argv[2])
    else:
        show(sys.argv[2])
