"""Summarise BM_PHASE_DUMP of the persistent kernel (task 20, every CTA)."""
import sys

import numpy as np

rows = [list(map(int, l.split()))[1:17] for l in open(sys.argv[1]) if l[0].isdigit()]
a = np.array(rows, dtype=np.float64)
names = {1: "header seen + grid barrier passed", 2: "row table built", 3: "first stage handed to MMA",
         4: "all MMAs done", 5: "TMEM->smem done (chunk 0)", 6: "cluster barrier A passed",
         7: "reduce+gates+scatter done", 8: "cluster barrier B passed", 9: "arrive at grid barrier"}
t0 = a[:, 0]
print("CTAs", len(a), " (times in us from the control thread starting to poll task 20)")
for k in range(1, 10):
    d = (a[:, k] - t0) / 1e3
    ok = a[:, k] > 0
    if not ok.any():
        continue
    print("  %-36s min %6.2f med %6.2f max %6.2f" % (names[k], d[ok].min(), np.median(d[ok]), d[ok].max()))
