"""Per kernel class (include/bm.h BM_K_*): DRAM bytes, L2->SM bytes, duration and tensor-pipe
activity per launch from an `ncu --set full` capture taken INSIDE a bench.py workload, plus the
class shares of the ncu launch list of the same command. Writes profiles/round*/traffic_<wl>.json,
which bench.py reports as roofline.traffic (per class) for that workload.

usage: python tools/traffic_classes.py RAW.csv LAUNCHES.csv OUT.json "command description"
"""
import collections
import csv
import json
import re
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "usecond": 1, "nsecond": 1e-3, "msecond": 1e3}
EPI_CLASS = {0: 1, 1: 4, 2: 2, 3: 3}   # cell_step_sm100_kernel<EPI, ...> -> BM_K_*


def kclass(name):
    if "cell_pair2_kernel" in name or "cell_pair_kernel" in name:
        return 0
    m = re.search(r"cell_step_sm100_kernel<\(?(?:int)?\)?(\d+)", name)
    if m:
        return EPI_CLASS[int(m.group(1))]
    if "simt" in name:
        return 5
    return None


raw_csv, launches_csv, out, what = sys.argv[1:5]
rows = list(csv.reader(open(raw_csv)))
hdr, units, data = rows[0], rows[1], [r for r in rows[2:] if len(r) == len(rows[0])]


def get(d, m):
    i = hdr.index(m)
    try:
        return float(d[i].replace(",", "")) * UNIT.get(units[i], 1)
    except ValueError:
        return float("nan")


per = collections.defaultdict(list)
for d in data:
    k = kclass(d[hdr.index("Kernel Name")])
    if k is None:
        continue
    per[k].append({"dram": get(d, "dram__bytes_read.sum") + get(d, "dram__bytes_write.sum"),
                   "l2_to_sm": get(d, "l1tex__m_xbar2l1tex_read_bytes.sum"),
                   "us": get(d, "gpu__time_duration.sum"),
                   "tensor_pct": get(d, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"),
                   "grid": d[hdr.index("Grid Size")]})
lines = [l for l in open(launches_csv) if not l.startswith("==")]
lr = list(csv.reader(lines))
lh = lr[0]
cnt, tsum = collections.Counter(), collections.Counter()
for r in lr[1:]:
    if len(r) != len(lh):
        continue
    dd = dict(zip(lh, r))
    k = kclass(dd.get("Kernel Name", ""))
    if k is None:
        continue
    cnt[k] += 1
    try:
        tsum[k] += float(dd["Metric Value"].replace(",", ""))
    except (KeyError, ValueError):
        pass
tot_t = sum(tsum.values()) or 1.0
doc = {"what": what,
       "method": "ncu --set full (default cache control: caches flushed before every replay, so DRAM bytes are "
                 "cold-cache; inside the step the LSTM / tree weights stay L2-resident) of launches sampled inside "
                 "the command; launch list = ncu --metrics gpu__time_duration.sum --clock-control none of the same "
                 "command (serialised, cold: compare shares, not absolutes)",
       "classes": {}}
for k in sorted(set(per) | set(cnt)):
    v = per.get(k, [])
    n = len(v)
    doc["classes"][str(k)] = {
        "captured_launches": n,
        "dram_bytes_per_launch": sum(x["dram"] for x in v) / n if n else None,
        "l2_to_sm_bytes_per_launch": sum(x["l2_to_sm"] for x in v) / n if n else None,
        "ncu_us_per_launch": sum(x["us"] for x in v) / n if n else None,
        "tensor_pipe_pct": sum(x["tensor_pct"] for x in v) / n if n else None,
        "grids": sorted({x["grid"] for x in v}),
        "launch_list_count": cnt.get(k, 0),
        "launch_list_time_share": tsum.get(k, 0) / tot_t,
    }
json.dump(doc, open(out, "w"), indent=1)
print(json.dumps(doc, indent=1))
