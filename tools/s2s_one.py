"""Recompute chosen requests of a full-size configs[2] run (n requests at `rate`) with the
fp64 oracle (forced tokens) and the bf16-activation emulation; per layer errors. Tool only."""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from oracle import cells  # noqa: E402
from paper_conf_eurosys_gaoywl18_b200 import bm  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from s2s_diag import emulate  # noqa: E402

n, rate = int(sys.argv[1]), float(sys.argv[2])
reqs = [int(x) for x in sys.argv[3].split(",")]
w = bench.make_weights("seq2seq")
e, cellmap = bench.build_engine(bm, "seq2seq", w, 0, max_requests=n + 64, lookahead=1, time_kernels=0, keep=1)
trace = bench.make_trace("seq2seq", n, rate, 1000)
first = e.submit_many(e.prepare_requests(trace, cellmap))
assert e.run() == n
e.poll(n + 16)
hh = np.zeros((n, 4, 1024), np.float32)
cc = np.zeros((n, 4, 1024), np.float32)
toks = np.zeros((n, 340), np.int32)
e.read_results_many(first, n, h=hh, c=cc, tokens=toks, release=False)
from threadpoolctl import threadpool_limits
for r in reqs:
    q = trace[r]
    f = toks[r, :q.decode_len]
    with threadpool_limits(limits=os.cpu_count()):
        o = cells.seq2seq(w["enc"], w["dec"], q.tokens, q.decode_len, forced_tokens=f)
        eh, ec = emulate(w["enc"], w["dec"], q.tokens, f)
    print(json.dumps({"req": r, "src": len(q.tokens), "tgt": q.decode_len,
                      "dev_vs_oracle_h": [float(np.max(np.abs(hh[r, l] - o["h"][l]))) for l in range(4)],
                      "dev_vs_oracle_c": [float(np.max(np.abs(cc[r, l] - o["c"][l]))) for l in range(4)],
                      "dev_vs_emul_h": [float(np.max(np.abs(hh[r, l] - eh[l]))) for l in range(4)],
                      "dev_vs_emul_c": [float(np.max(np.abs(cc[r, l] - ec[l]))) for l in range(4)],
                      "emul_vs_oracle_c": [float(np.max(np.abs(ec[l] - o["c"][l]))) for l in range(4)],
                      "argmax_gap_max": float(max(o["logits"][s].max() - o["logits"][s][f[s]] for s in range(len(f)))),
                      "worst_c_unit_l0": int(np.argmax(np.abs(cc[r, 0] - o["c"][0])))}), flush=True)
