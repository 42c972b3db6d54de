"""Per-launch DRAM traffic of the LSTM cell-step kernels from `ncu --set full` captures taken
inside bench.py (tools/profile_round.sh), weighted by the kernels' launch counts in the ncu
launch list of the same bench command. Writes the JSON that bench.py reports as
roofline.traffic (bytes per launch, like roofline.achieved).

usage: python tools/traffic_from_ncu.py TAG OUT.json   (reads gpurun_out/*_TAG*)"""
import collections
import csv
import json
import sys

tag, out = sys.argv[1], sys.argv[2]
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def raw(k):
    rows = list(csv.reader(open(f"gpurun_out/prof_{k}_{tag}_raw.csv")))
    hdr, units, data = rows[0], rows[1], rows[2:]

    def get(d, m):
        return float(d[hdr.index(m)]) * UNIT.get(units[hdr.index(m)], 1)
    dram = [get(d, "dram__bytes_read.sum") + get(d, "dram__bytes_write.sum") for d in data]
    xbar = [get(d, "l1tex__m_xbar2l1tex_read_bytes.sum") for d in data]
    return sum(dram) / len(dram), sum(xbar) / len(xbar), len(data)


lines = [l for l in open(f"gpurun_out/launches_{tag}.csv") if not l.startswith("==")]
rows = list(csv.reader(lines))
hdr = rows[0]
count = collections.Counter()
for r in rows[1:]:
    if len(r) == len(hdr):
        name = dict(zip(hdr, r))["Kernel Name"]
        for k in ("cell_pair_kernel", "cell_step_sm100_kernel"):
            if k in name:
                count[k] += 1
res = {k: raw(k) for k in count}
n = sum(count.values())
doc = {
    "dram_bytes_per_launch": sum(count[k] * res[k][0] for k in count) / n,
    "l2_to_sm_bytes_per_launch": sum(count[k] * res[k][1] for k in count) / n,
    "per_kernel": {k: {"launch_share": count[k] / n, "dram_bytes": res[k][0], "l2_to_sm_bytes": res[k][1],
                       "captured_launches": res[k][2]} for k in count},
    "source": f"ncu --set full (default cache control: L2 flushed before each replay, so DRAM bytes are "
              f"cold-cache) of 3 launches per kernel inside bench.py (tools/profile_round.sh, tag {tag}); "
              f"weights = launch counts in the ncu launch list of bench.py --steps 2 --warmup 1",
}
json.dump(doc, open(out, "w"), indent=1)
print(json.dumps(doc, indent=1))
