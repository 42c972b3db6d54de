import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
import bench
from paper_conf_eurosys_gaoywl18_b200 import bm
wl = sys.argv[1]; run = int(sys.argv[2])
w = bench.make_weights(wl)
e, cells = bench.build_engine(bm, wl, w, 0, max_requests=2000, lookahead=1, time_kernels=1)
print("e ok", flush=True)
if run:
    trace = bench.make_trace(wl, 200, 20000.0, 1000)
    prep = e.prepare_requests(trace, cells)
    e.submit_many(prep); print("run", e.run(), flush=True)
e2, cells2 = bench.build_engine(bm, wl, w, 0, max_requests=2000, lookahead=1, time_kernels=0, keep=1)
print("e2 ok", flush=True)
