"""Per-launch DRAM traffic of a workload's cell-step kernels (seq2seq / tree) from one
`ncu --set full` capture of a sample of their launches inside bench.py, weighted by each
kernel's (name + template arguments) launch count in the ncu launch list of the same bench
command. Writes the JSON that bench.py reports as roofline.traffic for that workload.

usage: python tools/traffic_wl.py TAG WL OUT.json   (reads gpurun_out/{launches,prof}_WL_TAG*)"""
import collections
import csv
import json
import re
import sys

tag, wl, out = sys.argv[1], sys.argv[2], sys.argv[3]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
CELL = ("cell_pair_kernel", "cell_step_sm100_kernel")


def key(name):
    """kernel base name + template arguments (EPI_LSTM / EPI_PROJ / ... are template args)"""
    m = re.search(r"(cell_pair_kernel|cell_step_sm100_kernel)(<[^>]*>)?", name)
    return (m.group(1) + (m.group(2) or "")) if m else None


rows = list(csv.reader(open(f"gpurun_out/prof_{wl}_{tag}_raw.csv")))
hdr, units, data = rows[0], rows[1], rows[2:]


def get(d, m):
    return float(d[hdr.index(m)]) * UNIT.get(units[hdr.index(m)], 1)


cap = collections.defaultdict(list)
for d in data:
    k = key(d[hdr.index("Kernel Name")])
    if k:
        cap[k].append((get(d, "dram__bytes_read.sum") + get(d, "dram__bytes_write.sum"),
                       get(d, "l1tex__m_xbar2l1tex_read_bytes.sum"), get(d, "gpu__time_duration.sum")))
lines = [l for l in open(f"gpurun_out/launches_{wl}_{tag}.csv") if not l.startswith("==")]
lr = list(csv.reader(lines))
count, tsum = collections.Counter(), collections.Counter()
for r in lr[1:]:
    if len(r) == len(lr[0]):
        d = dict(zip(lr[0], r))
        k = key(d["Kernel Name"])
        if k and k in cap:
            count[k] += 1
            tsum[k] += float(d["Metric Value"])
n = sum(count.values())
per = {k: {"launch_share": count[k] / n, "time_share": tsum[k] / sum(tsum.values()),
           "dram_bytes": sum(x[0] for x in cap[k]) / len(cap[k]),
           "l2_to_sm_bytes": sum(x[1] for x in cap[k]) / len(cap[k]),
           "captured_launches": len(cap[k])} for k in count}
doc = {"dram_bytes_per_launch": sum(count[k] * per[k]["dram_bytes"] for k in count) / n,
       "l2_to_sm_bytes_per_launch": sum(count[k] * per[k]["l2_to_sm_bytes"] for k in count) / n,
       "per_kernel": per,
       "source": f"ncu --set full (L2 flushed before each replay: cold-cache DRAM bytes) of sampled cell-step "
                 f"launches inside bench.py --workload {wl} (tools/profile_wl.sh, tag {tag}); weights = launch "
                 f"counts in the ncu launch list of the same command"}
json.dump(doc, open(out, "w"), indent=1)
print(json.dumps(doc, indent=1))
