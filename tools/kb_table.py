"""Print a kbench log as one line per b: us per call and, per kernel class, device span and TFLOP/s."""
import json
import sys

for l in open(sys.argv[1]):
    if l.startswith("{"):
        d = json.loads(l)
        ks = [k for k in d if k.startswith("k")]
        print(d["cell"], d["b"], round(d["us_per_call"], 2),
              [(k, round(d[k]["span_us"], 2), round(d[k]["TFLOPs"]), round(d[k]["GBps"])) for k in ks])
