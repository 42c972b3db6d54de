"""Kernel micro-benchmark: one batched cell step (bm_cell_step, async) at fixed b, timed with
CUDA events on the engine stream over many back-to-back launches. Reports us/launch,
algorithmic GB/s and TFLOP/s per b. Used for the roofline sweep and under ncu."""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cell", default="lstm", choices=["lstm", "leaf", "internal", "proj"])
    ap.add_argument("--b", default="1,16,64,128,256,512")
    ap.add_argument("--iters", type=int, default=200)
    ap.add_argument("--fp32", action="store_true")
    ap.add_argument("--vary-tokens", type=int, default=0,
                    help="cycle through N row sets with fresh random tokens (embedding rows not L2-resident)")
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import torch
    from paper_conf_eurosys_gaoywl18_b200 import bm
    from workloads import gen
    H, V = 1024, 32768
    prec = bm.PREC_FP32 if a.fp32 else bm.PREC_BF16
    bf = not a.fp32
    pk = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                     "MEASURED_PEAKS.json")))
    e = bm.Engine(precision=prec, hidden=H, pool_layers=1, max_slots=8192, max_requests=8192,
                  max_decode_len=4, time_kernels=1, roof_hbm_gbs=pk["hbm_gbs"],
                  roof_tc_tflops=pk["bf16_tflops"])
    if a.cell in ("lstm", "proj"):
        w = gen.lstm_stack_weights(H, 1, V, 0, projection=a.cell == "proj", bf16=bf)
        kind = bm.CELL_LSTM_PROJ if a.cell == "proj" else bm.CELL_LSTM
        cid = e.load_cell(kind, 1, V, 512, 0, w.W, w.b, w.E, w.W_out, w.b_out)
        G, K, rows_w = 4, 2 * H, 4 * H
    else:
        t = gen.tree_weights(H, V, 0, bf16=bf)
        leaf = e.load_cell(bm.CELL_TREE_LEAF, 1, V, 512, 0, [t.W_leaf], [t.b_leaf], t.E)
        intern = e.load_cell(bm.CELL_TREE_INTERNAL, 1, V, 512, 1, [t.U], [t.b_int])
        cid = leaf if a.cell == "leaf" else intern
        G, K = (3, H) if a.cell == "leaf" else (5, 2 * H)
        rows_w = G * H
    stream = torch.cuda.ExternalStream(e.stream())
    rng = np.random.default_rng(0)
    out = []
    el = 2 if bf else 4
    for b in [int(x) for x in a.b.split(",")]:
        slots = rng.choice(8192, size=b, replace=False).astype(np.int32)
        if a.cell == "internal":
            kids = rng.choice(8192, size=2 * b, replace=False).astype(np.int32)
            rows = np.stack([kids[:b], kids[b:], slots, np.zeros(b)], 1)
        else:
            toks = rng.integers(3, V, size=b)
            rows = np.stack([toks, np.zeros(b), slots, (np.arange(b) % 2) * bm.ROW_PARITY], 1)
        row_sets = [rows]
        if a.vary_tokens and a.cell != "internal":
            row_sets = [np.stack([rng.integers(3, V, size=b), np.zeros(b), slots,
                                  (np.arange(b) % 2) * bm.ROW_PARITY], 1) for _ in range(a.vary_tokens)]
        for i in range(5):
            e.cell_step(cid, row_sets[i % len(row_sets)], sync=False)
        torch.cuda.synchronize()
        e.reset_stats()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        import time as _t
        th0 = _t.perf_counter()
        for i in range(a.iters):
            e.cell_step(cid, row_sets[i % len(row_sets)], sync=False)
        th1 = _t.perf_counter()
        ev1.record(stream)
        ev1.synchronize()
        us = ev0.elapsed_time(ev1) * 1e3 / a.iters
        st = e.stats()
        reps = int(os.environ.get("BM_REPEAT", "1"))
        # every launch's device span (first CTA past its dependency wait .. last CTA done) and
        # its algorithmic bytes / flops, per kernel class (include/bm.h "measurement")
        r = {"cell": a.cell, "b": b, "us_per_call": us, "us_per_step": us / reps,
             "host_us_per_call": (th1 - th0) * 1e6 / a.iters}
        for k in range(bm.K_CLASSES):
            n = st["k_launches"][k]
            if not n:
                continue
            span = st["k_span_ms"][k] / max(1, st["k_span_launches"][k])
            r[f"k{k}"] = {"launches": n, "span_us": span * 1e3,
                          "GBps": st["k_bytes"][k] / n / (span / 1e3) / 1e9,
                          "TFLOPs": st["k_flops"][k] / n / (span / 1e3) / 1e12,
                          "frac_binding_burst": st["k_roof_ms"][k] / st["k_span_ms"][k]}
        print(json.dumps(r), flush=True)
        out.append(r)
    if a.out:
        json.dump(out, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
