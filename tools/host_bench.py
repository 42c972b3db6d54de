"""Host-side cost of the C++ scheduler (no GPU: BM_CLOCK_DRY, Algorithm 1 + request processor +
slot pool + retire, one tick per task): ns per scheduled node and per task on a configs[1]-shaped
trace (WMT lengths, bmax 512, MaxTasksToSubmit 5, look-ahead k = 2). Arrivals are spaced so that
tasks carry ~350-450 rows, as in the GPU bench at its p90-bound rate."""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    from paper_conf_eurosys_gaoywl18_b200 import bm
    from workloads import gen
    n = int(os.environ.get("N", "20000"))
    per_tick = float(os.environ.get("PER_TICK", "16"))
    H = 64
    e = bm.Engine(clock=bm.CLOCK_DRY, hidden=H, max_slots=1 << 16, max_requests=n + 64,
                  schedule_when_outstanding_leq=2, record_log=0)
    W = [np.zeros((4 * H, 2 * H), np.float32)]
    cid = e.load_cell(bm.CELL_LSTM, 1, 32768, 512, 0, W, [np.zeros(4 * H, np.float32)],
                      np.zeros((32768, H), np.float32))
    trace = gen.chain_trace(n, 32768, 1000)
    for i, q in enumerate(trace):
        q.arrival = i / per_tick
    prep = e.prepare_requests(trace, {gen.CHAIN: (cid, 0)})
    e.submit_many(prep)
    t0 = time.perf_counter()
    assert e.run() == n
    wall = time.perf_counter() - t0
    st = e.stats()
    rows, tasks = st["rows"], st["tasks"]
    print(json.dumps({"requests": n, "tasks": tasks, "rows_per_task": rows / tasks,
                      "sched_ns_per_task": st["sched_ns"] / tasks, "sched_ns_per_node": st["sched_ns"] / rows,
                      "retire_ns_per_task": st["retire_ns"] / tasks, "launch_ns_per_task": st["launch_ns"] / tasks,
                      "run_wall_ns_per_node": wall * 1e9 / rows}))


if __name__ == "__main__":
    main()
