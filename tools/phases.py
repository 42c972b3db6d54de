"""Summarise BM_PHASE_DUMP files: per-phase durations (us) over the CTAs of each step.
Phases: 0 start, 1 setup done, 2 MMA done (main loop), 3 cluster barrier 1, 4 reduce+epilogue,
5 final cluster barrier."""
import sys

import numpy as np

steps = []
cur = None
for line in open(sys.argv[1]):
    if line.startswith("step"):
        cur = {"hdr": line.strip(), "rows": []}
        steps.append(cur)
    else:
        v = [int(x) for x in line.split()]
        cur["rows"].append(v[1:65] + [0] * (65 - len(v)))
for st in steps[-3:]:
    a = np.array(st["rows"], dtype=np.float64)
    t0 = a[:, 0].min()
    print(st["hdr"], "ctas", len(a), "span_us %.2f" % ((a[:, 5].max() - t0) / 1e3))
    names = ["start", "setup", "mainloop", "bar1", "reduce", "bar2"]
    print("  start offsets us: min %.2f med %.2f max %.2f" % tuple((np.percentile(a[:, 0] - t0, q) / 1e3) for q in (0, 50, 100)))
    for k in range(1, 6):
        d = (a[:, k] - a[:, k - 1]) / 1e3
        print("  %-8s us: min %.2f med %.2f max %.2f" % (names[k], d.min(), np.median(d), d.max()))
    for k, nm in ((8, "producer after PDL wait"), (9, "producer row table done"),
                  (10, "producer stage 0 issued"), (11, "producer first hand-off"),
                  (12, "second stage at MMA"), (13, "MMA got weight chunk 0"),
                  (6, "first stage at MMA (from setup)"), (7, "last stage at MMA (from setup)")):
        d = (a[:, k] - a[:, 1]) / 1e3
        print("  %-32s us: min %.2f med %.2f max %.2f" % (nm, d.min(), np.median(d), d.max()))
    if a.shape[1] >= 32 and a[:, 16].any():
        st = [np.median(a[:, 16 + k] - a[:, 1]) / 1e3 for k in range(12) if a[:, 16 + k].all()]
        wc = [np.median(a[:, 28 + k] - a[:, 1]) / 1e3 for k in range(4) if a[:, 28 + k].all()]
        print("  stage kb at MMA (med, from setup) us: " + " ".join("%.2f" % x for x in st))
        print("  weight chunk at MMA (med, from setup) us: " + " ".join("%.2f" % x for x in wc))
    if a.shape[1] >= 48 and a[:, 32].any():
        rp = [np.median(a[:, 32 + k] - a[:, 3]) / 1e3 for k in range(16) if a[:, 32 + k].all()]
        print("  reduce pass k start (med, from bar1 end) us: " + " ".join("%.2f" % x for x in rp))
    cyc = a[:, 15] - a[:, 14]
    ns = a[:, 5] - a[:, 0]
    ok = (cyc > 0) & (ns > 0)
    if ok.any():
        print("  SM clock (clock64 / globaltimer over each CTA): median %.0f MHz" % np.median(cyc[ok] / ns[ok] * 1e3))
