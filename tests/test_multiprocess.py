"""Multi-rank (world_size 2, gloo, CPU) coverage of the request-sharded path:
weights broadcast once from rank 0, each rank drives its own engine (BM_CLOCK_DRY: the
scheduler, no GPU) over its own Poisson shard, and the end-of-run collectives (max over ranks,
latency gather) combine the results. The per-step path has no collective."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from oracle.scheduler import CHAIN, Replay
    from paper_conf_eurosys_gaoywl18_b200 import bm, shard
    from workloads import gen

    H, V = 64, 64
    # rank 0 owns the weights; the other ranks start from garbage and must receive them
    w = gen.lstm_stack_weights(H, 1, V, seed=0 if rank == 0 else 99)
    shard.broadcast_arrays([("W", w.W[0]), ("b", w.b[0]), ("E", w.E)], dist)
    digest = float(np.abs(w.W[0]).sum() + np.abs(w.E).sum())
    # every rank: its own engine over its own shard (different seed, same per-GPU load)
    trace = gen.chain_trace(60, V, shard.rank_seed(100, rank), rate=2.0)
    e = bm.Engine(clock=bm.CLOCK_DRY, hidden=H, max_slots=128, max_requests=128,
                  schedule_when_outstanding_leq=1)
    cid = e.load_cell(bm.CELL_LSTM, 1, V, 16, 0, w.W, w.b, w.E)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    n = e.run()
    comp = e.poll()
    lat = np.array([c.t_done - c.t_arrival for c in comp])
    # the shard's schedule is exactly the single-engine replay of that shard
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    rp = Replay([(16, 0)], max_slots=128, schedule_when_outstanding_leq=1).run(reqs)
    ok_replay = [(c.req_id, c.t_done) for c in comp] == [(r, float(t)) for r, t in rp.completions]
    total = shard.reduce_sum(float(n), dist)
    span = shard.reduce_max(float(max(c.t_done for c in comp)), dist)
    all_lat = shard.gather_samples(lat, dist)
    digests = [torch.zeros(1, dtype=torch.float64) for _ in range(world)]
    dist.all_gather(digests, torch.tensor([digest], dtype=torch.float64))
    if rank == 0:
        np.save(os.path.join(out_dir, "res.npy"), np.array([
            total, span, len(all_lat), float(ok_replay),
            float(all(abs(d.item() - digests[0].item()) < 1e-9 for d in digests))]))
    dist.barrier()
    dist.destroy_process_group()


def test_two_rank_sharding_gloo(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    total, span, n_lat, ok_replay, same_weights = np.load(tmp_path / "res.npy")
    assert total == 120                    # every request of every shard completed
    assert n_lat == 120                    # latency samples gathered from both ranks
    assert span > 0
    assert ok_replay == 1.0                # each shard == single-engine replay of the shard
    assert same_weights == 1.0             # broadcast gave every rank rank 0's weights


def test_rank_seeds_differ():
    from paper_conf_eurosys_gaoywl18_b200 import shard
    assert len({shard.rank_seed(1000, r) for r in range(8)}) == 8


def test_bench_product_path_two_ranks_dry(tmp_path):
    """The product bench path end to end on 2 ranks: plain `bench.py --gpus 2` re-launches itself
    under torch.distributed.run (one process per GPU), rank 0 broadcasts the weights, every rank
    runs its own engine over its own Poisson shard (BM_CLOCK_DRY here: the scheduler without a
    GPU, collectives on gloo), and rank 0 prints ONE line with n_gpus = 2."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = tmp_path / "line.json"
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--dry", "--quick",
                        "--steps", "1", "--warmup", "1", "--reqs", "600", "--no-cpu-baseline", "--out", str(out)],
                       capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["comm"]["world_size"] == 2
    assert line["comm"]["backend"] == "gloo" and line["comm"]["per_step_collectives"] == 0
    assert line["value"] > 0 and line["config"]["parallelism"] == "request-sharded x2"
    assert json.loads(out.read_text())["n_gpus"] == 2


def test_bench_refuses_mismatched_world(tmp_path):
    """--gpus N under a launcher with WORLD_SIZE != N fails loudly instead of printing a 1-GPU line."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "8", "--dry"],
                       capture_output=True, text=True, timeout=300, cwd=root, env=env)
    assert r.returncode != 0 and "WORLD_SIZE" in (r.stderr + r.stdout)
