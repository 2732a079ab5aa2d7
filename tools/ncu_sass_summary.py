"""Summarise an `ncu --page source --csv --print-source sass` export: total warp
instructions, and the hottest SASS lines by executed count and by stall samples."""
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hdr = rows[1]
    out = []
    for r in rows[2:]:
        if len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        try:
            d["exe"] = int(d["Instructions Executed"] or 0)
            d["smp"] = int(d["Warp Stall Sampling (All Samples)"] or 0)
            d["thr"] = float(d["Avg. Threads Executed"] or 0)
        except ValueError:
            continue
        out.append(d)
    return out


def main(path, top=40, mode="exe"):
    ins = load(path)
    tot = sum(d["exe"] for d in ins)
    smp = sum(d["smp"] for d in ins)
    print(f"warp instructions executed: {tot:,}   stall samples: {smp:,}")
    if mode == "seq":
        for i, d in enumerate(ins):
            if d["exe"] * 1000 >= tot or d["smp"] * 200 >= smp:
                print(f"{i:5d} {d['exe']:>12,} {d['smp']:>7} {d['thr']:5.1f}  {d['Source'].strip()[:90]}")
        return
    key = "exe" if mode == "exe" else "smp"
    for d in sorted(ins, key=lambda x: -x[key])[:top]:
        print(f"{d['exe']:>12,} {d['smp']:>7} {d['thr']:5.1f}  {d['Source'].strip()[:100]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40, sys.argv[3] if len(sys.argv) > 3 else "exe")
