"""Summarise an `ncu --metrics gpu__time_duration.sum --csv --log-file` launch list:
per kernel name the launch count, total and mean duration; optionally the last N
launches in order (what one step or one sync point of the island loop runs)."""
import csv
import sys
from collections import OrderedDict


def load(path):
    rows = [r for r in csv.reader(open(path)) if r and not r[0].startswith("==")]
    hdr = rows[0]
    ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    out = []
    for r in rows[1:]:
        if len(r) != len(hdr) or r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
            continue
        v = float(r[iv].replace(",", ""))
        u = r[iu]
        us = v / 1000.0 if u in ("ns", "nsecond") else (v if u in ("us", "usecond") else v * 1000.0)
        out.append((r[ik].split("(")[0][:80], us))
    return out


def main(path, tail=0):
    ls = load(path)
    agg = OrderedDict()
    for k, us in ls:
        c, t = agg.get(k, (0, 0.0))
        agg[k] = (c + 1, t + us)
    tot = sum(t for _, t in agg.values())
    print(f"{len(ls)} launches, {tot:.1f} us")
    for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{c:6d} x {t / c:10.2f} us = {t:10.1f} us ({100 * t / tot:5.1f}%)  {k}")
    for k, us in ls[-tail:] if tail else []:
        print(f"   {us:10.2f} us  {k}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0)
