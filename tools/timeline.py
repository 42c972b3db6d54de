"""Summarise a BM_TIMELINE file (one block per engine): per launch, the device time from the
first CTA past the PDL wait to the last CTA end ("busy"), the gap from the previous launch's end
to this launch's first CTA past the wait ("gap"), how early its CTAs started before that
("early"), and host-side figures (issue -> device start, device end -> host retire; these assume
%globaltimer and CLOCK_REALTIME share an epoch, which the printed offsets make checkable)."""
import sys

import numpy as np


def blocks(path):
    cur = None
    for line in open(path):
        if line.startswith("#"):
            cur = {"L": [], "R": {}}
            yield cur
        elif line.startswith("L "):
            cur["L"].append([int(x) for x in line.split()[1:]])
        elif line.startswith("R "):
            k, v = line.split()[1:]
            cur["R"][int(k)] = int(v)


def main():
    path = sys.argv[1]
    skip = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
    for blk in list(blocks(path)):
        a = np.array(blk["L"], dtype=np.float64)
        if len(a) < 4:
            continue
        a = a[int(len(a) * skip):]
        idx, b, host, start, wait, end = a[:, 0], a[:, 1], a[:, 2], a[:, 3], a[:, 4], a[:, 5]
        busy = (end - wait) / 1e3
        gap = (wait[1:] - end[:-1]) / 1e3
        early = (wait - start) / 1e3
        per = np.diff(end) / 1e3
        issue_lead = (start - host) / 1e3
        q = lambda x: "med %7.2f  p10 %7.2f  p90 %7.2f" % (np.median(x), np.percentile(x, 10), np.percentile(x, 90))
        print("launches %d  b med %d" % (len(a), np.median(b)))
        print("  end-to-end per launch us  " + q(per))
        print("  busy (wait..end) us       " + q(busy))
        print("  gap (prev end..wait) us   " + q(gap))
        print("  early (start..wait) us    " + q(early))
        print("  dev start - host issue us " + q(issue_lead))
        # one launch per task (single-layer cells): launch index == task sequence number
        lag = [(blk["R"][int(i)] - e) / 1e3 for i, e in zip(idx, end) if int(i) in blk["R"]]
        if lag:
            print("  host retire - dev end us  " + q(np.array(lag)))
        nxt = host[1:] - end[:-1]
        print("  next issue - dev end us   " + q(nxt / 1e3))


if __name__ == "__main__":
    main()
