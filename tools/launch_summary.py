"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per kernel/grid,
count, mean duration and share of the total. ncu serialises launches and runs them cold, so
compare SHARES, not absolute times (B200_PROFILING.md)."""
import collections
import csv
import sys

lines = [l for l in open(sys.argv[1]) if not l.startswith("==")]
rows = list(csv.reader(lines))
hdr = rows[0]
data = [dict(zip(hdr, r)) for r in rows[1:] if len(r) == len(hdr)]
by = collections.defaultdict(list)
for d in data:
    name = d["Kernel Name"].split("(")[0].split("::")[-1]
    by[(name, d["Grid Size"])].append(float(d["Metric Value"]) / 1e3)
tot = sum(sum(v) for v in by.values())
print(f"{'kernel':34s} {'grid':16s} {'n':>5s} {'mean_us':>9s} {'share':>7s}")
for k, v in sorted(by.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k[0][:34]:34s} {k[1]:16s} {len(v):5d} {sum(v)/len(v):9.2f} {sum(v)/tot*100:6.1f}%")
