"""Per-task cost of the whole engine path at a fixed batch size: n requests of equal length, all
arriving at t = 0, bmax = b, so every task carries b rows. Reports device time per task (CUDA
events around bm_run on the engine stream) for the per-task launch path and the persistent
weight-stationary kernel."""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--b", default="16,64,128,256,384,512")
    ap.add_argument("--steps", type=int, default=48)
    ap.add_argument("--persistent", default="0,1")
    a = ap.parse_args()
    import torch
    from paper_conf_eurosys_gaoywl18_b200 import bm
    from workloads import gen
    H, V = 1024, 32768
    w = gen.lstm_stack_weights(H, 1, V, 0)
    for pk in [int(x) for x in a.persistent.split(",")]:
        for b in [int(x) for x in a.b.split(",")]:
            e = bm.Engine(hidden=H, max_slots=4096, max_requests=4096, schedule_when_outstanding_leq=2,
                          persistent=pk, record_log=0, time_kernels=1)
            cid = e.load_cell(bm.CELL_LSTM, 1, V, b, 0, w.W, w.b, w.E)
            stream = torch.cuda.ExternalStream(e.stream())
            tr = gen.chain_trace(b, V, 1, lengths=[a.steps] * b, arrivals=[0.0] * b)
            prep = e.prepare_requests(tr, {gen.CHAIN: (cid, 0)})
            for _ in range(2):
                e.submit_many(prep)
                e.run()
                e.poll(b + 8)
            e.reset_stats()
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e.submit_many(prep)
            ev0.record(stream)
            e.run()
            ev1.record(stream)
            ev1.synchronize()
            e.poll(b + 8)
            st = e.stats()
            ms = ev0.elapsed_time(ev1)
            print(json.dumps({"persistent": pk, "b": b, "tasks": st["tasks"], "us_per_task": ms * 1e3 / st["tasks"],
                              "span_us_per_task": sum(st["k_span_ms"]) * 1e3 / max(1, sum(st["k_span_launches"])),
                              "sched_us_per_task": st["sched_ns"] / 1e3 / st["tasks"],
                              "launch_us_per_task": st["launch_ns"] / 1e3 / st["tasks"],
                              "retire_us_per_task": st["retire_ns"] / 1e3 / st["tasks"],
                              "tasks_per_call": st["tasks"] / max(1, st["schedule_calls"]),
                              "host_ms": st["sched_ns"] / 1e6, "dev_ms": ms}), flush=True)
            e.close()


if __name__ == "__main__":
    main()
