"""Two independent engines (two streams, disjoint pools) on one GPU issuing LSTM cell steps
alternately: does a second independent task in flight raise throughput over one stream's
back-to-back (PDL-chained) launches? Reports us per launch for 1 engine and for 2 engines."""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import torch
    from paper_conf_eurosys_gaoywl18_b200 import bm
    from workloads import gen
    H, V = 1024, 32768
    w = gen.lstm_stack_weights(H, 1, V, 0)
    engines = []
    for _ in range(2):
        e = bm.Engine(hidden=H, pool_layers=1, max_slots=8192, max_requests=8192, max_decode_len=4)
        cid = e.load_cell(bm.CELL_LSTM, 1, V, 512, 0, w.W, w.b, w.E)
        engines.append((e, cid))
    rng = np.random.default_rng(0)
    iters = int(os.environ.get("ITERS", "200"))
    for b in [int(x) for x in os.environ.get("BS", "64,128,256,384,512").split(",")]:
        slots = rng.choice(8192, size=b, replace=False).astype(np.int32)
        toks = rng.integers(3, V, size=b)
        rows = np.stack([toks, np.zeros(b), slots, (np.arange(b) % 2) * bm.ROW_PARITY], 1)
        res = {"b": b}
        for ne in (1, 2):
            for _ in range(5):
                for e, cid in engines[:ne]:
                    e.cell_step(cid, rows, sync=False)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for _ in range(iters):
                for e, cid in engines[:ne]:
                    e.cell_step(cid, rows, sync=False)
            torch.cuda.synchronize()
            res[f"us_per_launch_{ne}eng"] = (time.perf_counter() - t0) * 1e6 / (iters * ne)
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
