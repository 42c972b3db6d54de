"""Leader / peer phase summary of the CTA-pair kernel (BM_PHASE_DUMP, last step in the file)."""
import sys

import numpy as np

steps, cur = [], None
for line in open(sys.argv[1]):
    if line.startswith("step"):
        cur = []
        steps.append((line.strip(), cur))
    else:
        v = [int(x) for x in line.split()]
        cur.append(v[1:65])
hdr, rows = steps[-1]
a = np.array(rows, dtype=np.float64)
lead, peer = a[a[:, 16] > 0], a[a[:, 16] == 0]
print(hdr, "leaders", len(lead), "peers", len(peer))


def t(x, k):
    ok = x[:, k] > 0
    return np.median((x[ok, k] - x[ok, 1]) / 1e3) if ok.any() else float("nan")


for nm, k in [("after dep", 8), ("stage0 issued", 10), ("done", 2), ("barA", 3), ("reduce", 4), ("barB", 5)]:
    print("  %-14s lead %6.2f  peer %6.2f" % (nm, t(lead, k), t(peer, k)))
for nm, k0 in [("local full", 40), ("peer full", 44), ("local wchunk", 48), ("peer wchunk", 52)]:
    print("  %-14s lead " % nm + " ".join("%6.2f" % t(lead, k0 + i) for i in range(4)) +
          "   peer " + " ".join("%6.2f" % t(peer, k0 + i) for i in range(4)))
