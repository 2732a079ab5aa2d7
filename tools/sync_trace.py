"""Read a SPLIT_TRACE csv written by a trace build (SPLIT_TRACE_BUILD=1) of an island run
with M = 10: row 10 holds the sync-point tail stamps of a RUN segment (0 tail start,
1 elite step done, 2 grid sync, 3 export done, 4 worst sample sorted, 5 collection done,
6 grid sync, 7 worst slots done), row 15 the next segment's head (0 stall decided,
1 grid sync, 2 import done, 3 grid sync).  Prints the phase durations in us."""
import sys

rows = {}
for ln in open(sys.argv[1]).read().splitlines()[1:]:
    p = ln.split(",")
    rows[int(p[0])] = [int(x) for x in p[1:]]
t = rows[10]
names = ["elite step", "grid sync", "export", "worst sample", "collect", "grid sync", "worst sort"]
print("tail:", ", ".join(f"{n} {(t[i + 1] - t[i]) / 1e3:.1f}" for i, n in enumerate(names) if t[i + 1] and t[i]),
      f"| total {(t[7] - t[0]) / 1e3:.1f} us")
h = rows[15]
names = ["grid sync", "import", "grid sync"]
print("head:", ", ".join(f"{n} {(h[i + 1] - h[i]) / 1e3:.1f}" for i, n in enumerate(names) if h[i + 1] and h[i]),
      f"| total {(h[3] - h[0]) / 1e3:.1f} us")
g = rows[0]
print("generation 0 of the segment: lead_start..lead_end", (g[3] - g[0]) / 1e3, "us")
