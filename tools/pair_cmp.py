"""Run fixed LSTM steps (b = 129..512, random slots/states/flags, h = 1024) and save the result
rows and pool state to argv[1] (.npz), so two kernel variants (e.g. BM_PAIR2=0 / 1) can be
compared bit for bit. Tool only."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_gaoywl18_b200 import bm  # noqa: E402
from workloads import gen  # noqa: E402

h, V = 1024, 512
w = gen.lstm_stack_weights(h, 1, V, 5)
e = bm.Engine(hidden=h, pool_layers=1, max_slots=4096, max_requests=1024)
cid = e.load_cell(bm.CELL_LSTM, 1, V, 512, 0, w.W, w.b, w.E)
rng = np.random.default_rng(9)
out = {}
for b in (129, 160, 200, 256, 300, 384, 448, 512):
    slots = rng.choice(4096, size=b, replace=False).astype(np.int32)
    par = rng.integers(0, 2, size=b)
    first = rng.random(b) < 0.2
    h0 = gen.bf16_round(rng.uniform(-1, 1, (b, h)).astype(np.float32))
    c0 = rng.uniform(-2, 2, (b, h)).astype(np.float32)
    for p in (0, 1):
        m = par == p
        if m.any():
            e.pool_write(0, p, slots[m], h0[m], c0[m])
    toks = rng.integers(3, V, size=b)
    flags = (first * bm.ROW_FIRST) | bm.ROW_LAST | (par * bm.ROW_PARITY) | (np.arange(b) << 8)
    e.cell_step(cid, np.stack([toks, np.zeros(b), slots, flags], 1).astype(np.int32))
    rh, rc = e.result_rows(np.arange(b))
    out[f"h{b}"], out[f"c{b}"] = rh, rc
np.savez(sys.argv[1], **out)
if len(sys.argv) > 2:
    ref = np.load(sys.argv[2])
    worst = max(float(np.max(np.abs(out[k] - ref[k]))) for k in out)
    same = all(np.array_equal(out[k], ref[k]) for k in out)
    print({"bitwise_equal": same, "max_abs_diff": worst})
