"""Aggregate an `ncu --page source --csv --print-source cuda,sass` export per CUDA
source line: instructions executed and stall samples, hottest first."""
import csv
import sys


def main(path, top=40, div=1.0):
    rows = list(csv.reader(open(path)))
    hdr = None
    out = []
    for r in rows:
        if r and r[0] == "Line No":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr) or r[2] != "-":
            continue
        try:
            exe = int(r[7] or 0)
            smp = int(r[4] or 0)
        except ValueError:
            continue
        out.append((int(r[0]), r[1].strip(), exe, smp))
    tot = sum(x[2] for x in out)
    ts = sum(x[3] for x in out)
    print(f"instructions {tot:,}  samples {ts:,}  (per unit: {tot / div:,.1f})")
    for ln, src, exe, smp in sorted(out, key=lambda x: -x[2])[:top]:
        print(f"{ln:5d} {exe / div:9.1f} {100 * exe / tot:5.1f}% smp {100 * smp / max(ts, 1):5.1f}%  {src[:90]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40, float(sys.argv[3]) if len(sys.argv) > 3 else 1.0)
