"""One-screen summary of a bench.py JSON line: headline, e2e, per-kernel roofline, extras."""
import json
import sys

d = json.loads(open(sys.argv[1]).read())
print("value %.0f req/s  e2e %.0f  p90 %.2f ms  offered %.0f  achieved/offered %.3f  clocks %s" % (
    d["value"], d["e2e"]["value"] if d.get("e2e") else -1, d["latency_ms"]["p90"], d["config"]["offered_rate_per_gpu"],
    d.get("achieved_over_offered", 0), d.get("clocks")))
r = d["roofline"]
print("roofline: %s %s %.1f/%.1f %s frac %.3f binding %.3f kernel_ms/step %.1f ms/step %.1f" % (
    r["kernel"], r["bound"], r["achieved"], r["peak"], r["unit"], r["frac"], r["frac_binding"], r["kernel_ms_per_step"],
    d["ms_per_step"]))
for k, v in r["kernels"].items():
    print("  k%s %-45s n=%d rows %.0f span %.2f us frac %.3f binding %.3f share %.2f" % (
        k, v["name"], v["launches"], v["rows_per_launch"], v["span_us_per_launch"], v["frac"], v["frac_binding"],
        v["share_of_kernel_time"]))
for w, x in (d.get("extra_workloads") or {}).items():
    print("%s: %.0f req/s p90 %.2f ms offered %.0f" % (w, x["value"], x["latency_ms"]["p90"], x["offered_rate_per_gpu"]))
    for k, v in x["roofline"]["kernels"].items():
        print("  k%s n=%d rows %.0f span %.2f us frac %.3f share %.2f" % (
            k, v["launches"], v["rows_per_launch"], v["span_us_per_launch"], v["frac"], v["share_of_kernel_time"]))
if d.get("cpu_baseline"):
    print("cpu_baseline", d["cpu_baseline"]["value"], d["cpu_baseline"]["cores"])
