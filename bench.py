#!/usr/bin/env python
"""bench.py -- requests/sec at a p90-latency bound for cellular batching on B200.

Workload (BASELINE.json configs[1], the metric's configuration): 1-layer LSTM, h = 1024,
WMT-like sentence lengths (mean 24, max 330; L421, L635), Poisson open-loop arrivals (L423),
bmax 512 (L429), MaxTasksToSubmit 5 (L379), synthetic seeded weights/tokens.
`--workload seq2seq|tree` runs configs[2] / configs[3] instead.

A STEP = one open-loop Poisson trace of --reqs requests at the offered rate lambda* pushed
through the whole hot path (A1 unfold at admission, A2-A3 Algorithm 1, A4 slot pool, A5 launch,
A6-A9 fused gather/tcgen05/gate/scatter kernels, A12 completion signal, A13 poll/retire),
by the C-ABI engine's own event loop (bm_run). lambda* = the highest rate of a load sweep
(run first, untimed) whose p90 latency stays within the bound (--p90-ms, default 12 ms: the
paper's flat-region LSTM p90, L489).

value    = requests completed by all ranks / max over ranks of the device time of the K steps
e2e      = same, through the public API with host buffers: per step the bm_request arrays are
           submitted from host memory, row descriptors (tokens inside) go host->device from
           pinned memory on every Schedule call, and all final h rows come back device->host
roofline = the LSTM cell-step kernel: algorithmic bytes / CUDA-event time of every launch in
           the timed region, against MEASURED_PEAKS.json
Multi-GPU (torchrun): one engine per GPU, requests sharded by rank (weak scaling: each rank
runs its own lambda* Poisson stream), weights broadcast once from rank 0 with NCCL; no
collective on the per-step path.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

# the CPU oracle baseline forks one process per core: pin BLAS to one thread per process
# BEFORE numpy is imported (an inherited multi-threaded BLAS would oversubscribe the cores)
for _v in ("OMP_NUM_THREADS", "OPENBLAS_NUM_THREADS", "MKL_NUM_THREADS"):
    os.environ.setdefault(_v, "1")

import numpy as np  # noqa: E402

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from workloads import gen  # noqa: E402

METRIC = "requests/sec at p90-latency bound"


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--workload", default="lstm", choices=["lstm", "seq2seq", "tree"])
    p.add_argument("--reqs", type=int, default=0, help="requests per step (0 = per-workload default)")
    p.add_argument("--p90-ms", type=float, default=0.0,
                   help="p90 bound; 0 = per-workload default (12 ms, L489; Seq2Seq: the knee, "
                        "2x the lowest-load p90, since Fig. 13's values are not legible)")
    p.add_argument("--rate", type=float, default=0.0, help="skip the sweep, use this offered rate")
    p.add_argument("--lookahead", type=int, default=-1,
                   help="schedule when <= k tasks are outstanding (0 = the paper's idle-only); "
                        "-1 = per-workload default")
    p.add_argument("--persistent", type=int, default=-1,
                   help="1: persistent weight-stationary LSTM kernel (configs[1]); 0: one launch per "
                        "task; -1: per-workload default")
    p.add_argument("--policy", default="cellular", choices=["cellular", "graph"],
                   help="graph: the padding + bucketing graph-batching baseline of §7.1 (L427: bucket "
                        "width 10, round robin over buckets) on the same kernels (lstm workload only)")
    p.add_argument("--bucket-width", type=int, default=10)
    p.add_argument("--lengths", default="wmt", choices=["wmt", "fixed24", "clip50", "clip100", "identical"],
                   help="LSTM request lengths: WMT-like (configs[1]) or Fig. 11's variants (L643-L681); "
                        "tree: 'identical' = every request the complete 16-leaf tree (Fig. 15, L857)")
    p.add_argument("--enc-bmax", type=int, default=512,
                   help="Seq2Seq encoder bmax (decoder 256): 512 = BatchMaker-512,256, 256 = -256,256 (L717)")
    p.add_argument("--workers", type=int, default=1,
                   help="Algorithm 1 workers per GPU (one stream each, subgraph pinning, §8f N2)")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-seconds", type=float, default=15.0)
    p.add_argument("--out", default="")
    return p.parse_args()


# ------------------------------------------------------------------------------ workloads
WL = {
    "lstm": dict(config="BASELINE configs[1]: 1-layer LSTM h=1024, WMT-like lengths, Poisson arrivals, "
                        "bmax 512, 1 B200", hidden=1024, layers=1, vocab=32768, reqs=20000,
                 p90_ms=12.0, lookahead=2, persistent=0),
    "seq2seq": dict(config="BASELINE configs[2]: Seq2Seq 4+4 layer LSTM h=1024, vocab 32768, greedy "
                           "decode, encoder/decoder bmax 512/256", hidden=1024, layers=4, vocab=32768,
                    reqs=4000, p90_ms=None, lookahead=1, persistent=0),
    "tree": dict(config="BASELINE configs[3]: TreeLSTM h=1024, TreeBank-shaped binary trees, leaf/internal "
                        "cells batched separately, bmax 64", hidden=1024, layers=1, vocab=32768, reqs=6000,
                 p90_ms=12.0, lookahead=2, persistent=0),
}


ENC_BMAX = 512    # --enc-bmax (Seq2Seq encoder bmax; L717: BatchMaker-512,256 vs -256,256)
LENGTHS = "wmt"   # --lengths (LSTM): wmt | fixed24 | clip50 | clip100 (Fig. 11)


def chain_lengths(n, seed, kind):
    """Fig. 11's length mixes: the WMT-like distribution, every request 24 steps, or WMT clipped
    at 50 / 100 steps (L643-L667)."""
    if kind == "fixed24":
        return np.full(n, 24, np.int64)
    wmt = gen.wmt_lengths(n, np.random.default_rng(seed + 77))
    return np.minimum(wmt, {"clip50": 50, "clip100": 100}[kind])


def make_trace(wl, n, rate, seed):
    if wl == "lstm":
        lengths = None if LENGTHS == "wmt" else chain_lengths(n, seed, LENGTHS)
        return gen.chain_trace(n, WL[wl]["vocab"], seed, rate=rate, lengths=lengths)
    if wl == "seq2seq":
        return gen.seq2seq_trace(n, WL[wl]["vocab"], seed, rate=rate)
    return gen.tree_trace(n, WL[wl]["vocab"], seed, rate=rate, identical=LENGTHS == "identical")


def make_weights(wl):
    h, L, V = WL[wl]["hidden"], WL[wl]["layers"], WL[wl]["vocab"]
    if wl == "lstm":
        return {"cell": gen.lstm_stack_weights(h, L, V, seed=0)}
    if wl == "seq2seq":
        return {"enc": gen.lstm_stack_weights(h, L, V, seed=0),
                "dec": gen.lstm_stack_weights(h, L, V, seed=1, projection=True)}
    return {"tree": gen.tree_weights(h, V, seed=0)}


def weight_arrays(w):
    """Flat list of (name, ndarray) views of every weight array (for the NCCL broadcast)."""
    out = []
    for k, v in sorted(w.items()):
        for f in ("W", "b"):
            if hasattr(v, f):
                for i, a in enumerate(getattr(v, f)):
                    out.append((f"{k}.{f}{i}", a))
        for f in ("E", "W_out", "b_out", "W_leaf", "b_leaf", "U", "b_int"):
            a = getattr(v, f, None)
            if a is not None:
                out.append((f"{k}.{f}", a))
    return out


# ------------------------------------------------------------------------------ engine
def build_engine(bm, wl, w, device, max_requests, lookahead, time_kernels=1, keep=0, persistent=0,
                 policy=0, bucket_width=10, workers=1):
    h, L, V = WL[wl]["hidden"], WL[wl]["layers"], WL[wl]["vocab"]
    e = bm.Engine(device=device, hidden=h, pool_layers=L, max_slots=1 << 16, max_requests=max_requests,
                  schedule_when_outstanding_leq=lookahead, time_kernels=time_kernels, keep_results=keep,
                  max_decode_len=340, record_log=0, persistent=persistent, policy=policy,
                  bucket_width=bucket_width, workers=workers)
    if wl == "lstm":
        c = w["cell"]
        cid = e.load_cell(bm.CELL_LSTM, L, V, 512, 0, c.W, c.b, c.E)
        cells = {gen.CHAIN: (cid, 0)}
    elif wl == "seq2seq":
        enc, dec = w["enc"], w["dec"]
        ce = e.load_cell(bm.CELL_LSTM, L, V, ENC_BMAX, 0, enc.W, enc.b, enc.E)
        cd = e.load_cell(bm.CELL_LSTM_PROJ, L, V, 256, 1, dec.W, dec.b, dec.E, dec.W_out, dec.b_out)
        cells = {gen.SEQ2SEQ: (ce, cd)}
    else:
        t = w["tree"]
        lf = e.load_cell(bm.CELL_TREE_LEAF, 1, V, 64, 0, [t.W_leaf], [t.b_leaf], t.E)
        it = e.load_cell(bm.CELL_TREE_INTERNAL, 1, V, 64, 1, [t.U], [t.b_int])
        cells = {gen.TREE: (lf, it)}
    return e, cells


def run_trace(e, prepared, n):
    """Submit a prepared trace and drive it to completion; returns (wall s, latencies s)."""
    e.submit_many(prepared)
    t0 = time.perf_counter()
    done = e.run()
    t1 = time.perf_counter()
    comp = e.poll_array(n + 16)
    assert done == n and len(comp) == n, (done, len(comp), n)
    lat = comp["t_done"] - comp["t_arrival"]
    return t1 - t0, lat


def pct(a, q):
    return float(np.percentile(a, q)) if len(a) else float("nan")


def load_traffic(wl="lstm"):
    """roofline.traffic: per-launch DRAM bytes of the workload's cell-step kernels from the newest
    committed ncu summary (LSTM: profiles/round*/traffic_r*.json, tools/traffic_from_ncu.py;
    seq2seq / tree: profiles/round*/traffic_<wl>_*.json, tools/traffic_wl.py)."""
    import glob
    pat = "traffic_r*.json" if wl == "lstm" else f"traffic_{wl}_*.json"
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "round*", pat)))
    if not files:
        return None
    d = json.load(open(files[-1]))
    d["file"] = os.path.relpath(files[-1], ROOT)
    return d


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled DURING the timed region."""

    def __init__(self, device):
        self.device = device
        self.samples = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), "--query-gpu=clocks.sm,clocks.max.sm,power.draw,"
                 "clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
                 "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                 "clocks_event_reasons.sw_power_cap", "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm = [float(s[0]) for s in self.samples if len(s) >= 8 and s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if len(s) >= 8 and s[1].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for s in self.samples:
            if len(s) >= 8:
                for i, n in enumerate(names):
                    if s[4 + i].lower() == "active":
                        reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------ CPU oracle
def _oracle_worker(args):
    os.environ["OMP_NUM_THREADS"] = "1"
    wl, idx, seed, n = args
    from oracle import cells
    w = make_weights(wl)
    trace = make_trace(wl, n, None, seed)
    t0 = time.perf_counter()
    for i in idx:
        q = trace[i]
        if wl == "lstm":
            cells.chain_lstm(w["cell"], q.tokens)
        elif wl == "seq2seq":
            cells.seq2seq(w["enc"], w["dec"], q.tokens, q.decode_len)
        else:
            cells.tree_lstm(w["tree"], q.tokens, q.left, q.right)
    return len(idx), time.perf_counter() - t0


def _cost(q):
    """Cell steps of one request (the oracle's work unit)."""
    return len(q.tokens) + q.decode_len if q.left is None else len(q.left)


def cpu_oracle(wl, seconds, seed=1000):
    """The fp64 oracle (unbatched, step by step) on the host cores over a bounded sample of the
    same generated requests: one process per core, BLAS pinned to one thread. The sample is the
    first requests of the trace whose total cell steps fit ~`seconds` of work per core."""
    import multiprocessing as mp
    cores = os.cpu_count() or 1
    trace = make_trace(wl, 20000, None, seed)
    # calibrate the cost of one cell step on this host
    probe = [i for i in range(len(trace)) if _cost(trace[i]) >= 8][:1]
    n_est, dt = _oracle_worker((wl, probe, seed, 20000))
    per_step = dt / _cost(trace[probe[0]])
    budget = seconds * cores / per_step
    idx, tot = [], 0
    for i, q in enumerate(trace):
        if tot + _cost(q) > budget and idx:
            break
        idx.append(i)
        tot += _cost(q)
    chunks = [idx[c::cores] for c in range(cores)]
    ctx = mp.get_context("fork")
    t0 = time.perf_counter()
    with ctx.Pool(cores) as pool:
        res = pool.map(_oracle_worker, [(wl, ch, seed, 20000) for ch in chunks if ch])
    wall = time.perf_counter() - t0
    done = sum(r[0] for r in res)
    return {"value": done / wall, "unit": "requests/sec", "cores": cores, "kind": "oracle",
            "sample": f"first {done} requests ({tot} cell steps) of the {wl} trace generator "
                      f"(seed {seed}), fp64 numpy, closed loop, {cores} processes x 1 BLAS thread, "
                      f"{wall:.1f} s wall"}


# ------------------------------------------------------------------------------ reference arm
def reference_arm(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    wl = a.workload
    res = []
    for s in range(a.warmup + a.steps):
        r = cpu_oracle(wl, max(2.0, min(a.cpu_seconds, 10.0)), seed=1000 + s)
        if s >= a.warmup:
            res.append(r)
    v = float(np.mean([r["value"] for r in res]))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "requests/sec", "n_gpus": a.gpus,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": None, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": WL[wl]["config"]},
            "cpu_baseline": {"value": v, "unit": "requests/sec", "cores": res[0]["cores"], "kind": "oracle",
                             "sample": res[0]["sample"]},
            "e2e": {"value": v, "unit": "requests/sec", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ main arm
def main():
    global LENGTHS, ENC_BMAX
    a = parse()
    ENC_BMAX = a.enc_bmax
    LENGTHS = a.lengths if (a.workload == "lstm" and a.lengths != "identical") or \
        (a.workload == "tree" and a.lengths == "identical") else "wmt"
    if a.impl == "reference":
        return reference_arm(a)
    import torch
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    # one GPU per rank (NCCL over NVLink). With fewer GPUs than ranks (a functional check of the
    # multi-rank path on one GPU) ranks share devices and the few collectives go over gloo.
    ndev = max(1, torch.cuda.device_count())
    local = local_rank % ndev
    shared = world > ndev
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    coll_dev = None if shared else torch.device("cuda", local)
    from paper_conf_eurosys_gaoywl18_b200 import bm, shard

    wl = a.workload
    n_req = a.reqs or WL[wl]["reqs"]
    if a.lookahead < 0:
        a.lookahead = WL[wl]["lookahead"]
    if a.persistent < 0:
        a.persistent = WL[wl]["persistent"]
    policy = bm.POLICY_GRAPH if a.policy == "graph" else bm.POLICY_CELLULAR
    if policy == bm.POLICY_GRAPH and wl != "lstm":
        raise SystemExit("--policy graph: chain LSTM workload only (reading G5)")
    if policy == bm.POLICY_GRAPH:
        a.persistent = 0
    # ---- weights: generated on rank 0, broadcast once over NCCL (NVLink), never again
    w = make_weights(wl)
    if dist is not None:
        shard.broadcast_arrays(weight_arrays(w), dist, device=coll_dev)
    e, cells = build_engine(bm, wl, w, local, max_requests=max(n_req, 1 << 15) + 64, lookahead=a.lookahead,
                            persistent=a.persistent, policy=policy, workers=a.workers, bucket_width=a.bucket_width)
    stream = torch.cuda.ExternalStream(e.stream(), device=torch.device("cuda", local))

    def barrier():
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()

    def allmax(x):
        return shard.reduce_max(x, dist, device=coll_dev)

    # ---- calibrate saturation: every request of a trace arrives at t = 0
    burst = make_trace(wl, n_req, None, seed=shard.rank_seed(7, rank))
    pb = e.prepare_requests(burst, cells)
    run_trace(e, pb, n_req)                      # warm (also JIT of nothing: all AOT)
    dt, _ = run_trace(e, pb, n_req)
    mu = n_req / dt
    # ---- load sweep (open loop), untimed: highest rate whose p90 <= bound
    curve = []
    bound_kind = "absolute"
    if a.rate > 0:
        lam_star = a.rate
        bound_ms = a.p90_ms or WL[wl]["p90_ms"] or 12.0
    else:
        for frac in (0.05, 0.1, 0.2, 0.35, 0.5, 0.65, 0.8, 0.9, 1.0, 1.1):
            lam = frac * mu
            n_pt = int(max(2000, min(n_req, lam * 0.25)))
            tr = make_trace(wl, n_pt, lam, seed=shard.rank_seed(100, rank))
            p = e.prepare_requests(tr, cells)
            wall, lat = run_trace(e, p, n_pt)
            p50, p90, p99 = (allmax(pct(lat, q)) for q in (50, 90, 99))
            curve.append({"offered": lam, "achieved": n_pt / wall, "p50_ms": p50 * 1e3, "p90_ms": p90 * 1e3,
                          "p99_ms": p99 * 1e3})
        bound_ms = a.p90_ms or WL[wl]["p90_ms"]
        if not bound_ms:   # the knee: 2x the lowest-load p90
            bound_ms = 2.0 * curve[0]["p90_ms"]
            bound_kind = "knee (2x lowest-load p90)"

        def best_under(b):
            ok = [c["offered"] for c in curve if c["p90_ms"] <= b]
            return max(ok) if ok else None
        lam_star = best_under(bound_ms) or curve[0]["offered"]
        knee_ms = 2.0 * curve[0]["p90_ms"]
        bounds = {"12ms": best_under(12.0), "knee": best_under(knee_ms), "knee_ms": knee_ms}
    # ---- timed steps at lambda*
    trace = make_trace(wl, n_req, lam_star, seed=shard.rank_seed(1000, rank))
    prep = e.prepare_requests(trace, cells)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")   # > 126 MB L2
    for _ in range(a.warmup):
        run_trace(e, prep, n_req)
    e.reset_stats()
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    dev_ms = 0.0
    lats, queue, compute = [], [], []
    with ClockSampler(local) as clk:
        for _ in range(a.steps):
            flush.zero_()
            torch.cuda.synchronize()
            e.submit_many(prep)
            ev0.record(stream)
            done = e.run()
            ev1.record(stream)
            ev1.synchronize()
            assert done == n_req
            dev_ms += ev0.elapsed_time(ev1)
            comp = e.poll_array(n_req + 16)
            lats.append(comp["t_done"] - comp["t_arrival"])
            queue.append(comp["t_first"] - comp["t_arrival"])   # E5 (Fig. 9): queueing
            compute.append(comp["t_done"] - comp["t_first"])     # ... and computation time
    barrier()
    st = e.stats()
    lat = shard.gather_samples(np.concatenate(lats), dist, device=coll_dev)
    q_lat = shard.gather_samples(np.concatenate(queue), dist, device=coll_dev)
    c_lat = shard.gather_samples(np.concatenate(compute), dist, device=coll_dev)
    t_max = allmax(dev_ms / 1e3)
    total = n_req * a.steps * world
    value = total / t_max
    p50, p90, p99 = shard.percentiles(lat)   # over the union of all ranks' requests
    # ---- e2e: public API with host buffers (submit from host, descriptors H2D every Schedule
    #      call inside bm_run, final h rows D2H), timed on the host clock around the whole thing
    e2, cells2 = build_engine(bm, wl, w, local, max_requests=n_req + 64, lookahead=a.lookahead,
                              time_kernels=0, keep=1, persistent=a.persistent, policy=policy, workers=a.workers,
                              bucket_width=a.bucket_width)
    L, H = WL[wl]["layers"], WL[wl]["hidden"]
    hbuf = torch.empty((n_req, L, H), dtype=torch.float32).pin_memory().numpy()
    prep2 = e2.prepare_requests(trace, cells2)
    for _ in range(max(1, a.warmup)):
        fid = e2.submit_many(prep2)
        e2.run()
        e2.poll_array(n_req + 16)
        e2.read_results_many(fid, n_req, h=hbuf, release=True)
    barrier()
    t0 = time.perf_counter()
    rows0 = e2.stats()["rows"]
    ph = np.zeros(4)
    for _ in range(a.steps):
        tp = [time.perf_counter()]
        fid = e2.submit_many(prep2)
        tp.append(time.perf_counter())
        e2.run()
        tp.append(time.perf_counter())
        e2.poll_array(n_req + 16)
        tp.append(time.perf_counter())
        e2.read_results_many(fid, n_req, h=hbuf, release=True)
        tp.append(time.perf_counter())
        ph += np.diff(tp)
    e2e_s = allmax(time.perf_counter() - t0)
    rows_e2e = (e2.stats()["rows"] - rows0) / a.steps
    e2e = {"value": total / e2e_s, "unit": "requests/sec",
           "h2d_bytes_per_step": int(rows_e2e * 16),
           "d2h_bytes_per_step": int(n_req * L * H * 4),
           "host_ms_per_step": dict(zip(("submit", "run", "poll", "read_results"),
                                        (float(x) for x in ph * 1e3 / a.steps)))}
    # ---- roofline of the dominant kernel (the LSTM / tree cell step), live CUDA events
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    hbm = peaks.get("hbm_gbs", 6650.0)
    if st["timed_ms"] > 0:   # per-launch CUDA events (sampled launches) on the engine stream
        t_kern = st["timed_ms"]
        timing = ("CUDA events on the engine stream around a sample of cell-step launches (every 8th: "
                  "events between launches would disable PDL overlap)")
        kernel = {"lstm": "LSTM cell step: cell_pair_kernel (129-512 rows) + cell_step_sm100_kernel<EPI_LSTM>",
                  "seq2seq": "Seq2Seq cell steps: 4 LSTM layers (cell_pair_kernel / cell_step_sm100_kernel<EPI_LSTM>) "
                             "+ projection/argmax cell_step_sm100_kernel<EPI_PROJ>",
                  "tree": "TreeLSTM cell steps: cell_step_sm100_kernel<EPI_LEAF> + <EPI_INTERNAL>"}[wl]
    else:                    # persistent kernel: tasks run inside one launch
        t_kern = st["span_ms"]
        timing = ("persistent kernel: per-task device span (%globaltimer, first CTA ready .. last CTA "
                  "done, summed over every task of the timed region); CUDA events bracket each whole step")
        kernel = "lstm_persistent_kernel"
    achieved = st["timed_bytes"] / (t_kern / 1e3) / 1e9 if t_kern > 0 else 0.0
    tflops = st["timed_flops"] / (t_kern / 1e3) / 1e12 if t_kern > 0 else 0.0
    bf16_peak = peaks.get("bf16_tflops", 1590.0)
    traffic = load_traffic(wl) if not a.persistent else None
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
            "traffic": traffic["dram_bytes_per_launch"] if traffic else None,
            "traffic_unit": "bytes/launch (DRAM read+write, ncu, cold L2)",
            "traffic_l2_to_sm": traffic["l2_to_sm_bytes_per_launch"] if traffic else None,
            "traffic_source": traffic["file"] if traffic else None, "kernel": kernel, "timing": timing, "launches": st["timed_launches"],
            "avg_launch_us": t_kern * 1e3 / max(1, st["timed_launches"]),
            "avg_rows_per_task": st["rows"] / max(1, st["tasks"]), "tensor_tflops": tflops,
            "tensor_frac": tflops / bf16_peak,
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured copy)" if peaks else "fallback 6.65 TB/s",
            # the same sampled launches timed on the device (%globaltimer: first CTA past its
            # dependency wait .. last CTA done): excludes the serialisation the events impose
            "device_span_us": (st["span_ms"] * 1e3 / st["span_launches"]) if st["span_launches"] else None,
            "frac_device_span": ((st["timed_bytes"] / max(1, st["timed_launches"])) /
                                 (st["span_ms"] / 1e3 / st["span_launches"]) / 1e9 / hbm)
            if st["span_launches"] and st["timed_ms"] > 0 else None,
            "note": ("algorithmic bytes count the 16.8 MB weight stream per step even when the persistent "
                     "kernel keeps the weights on chip (so frac can exceed what DRAM moved)")}
    bound = None
    if wl == "lstm" and LENGTHS == "fixed24":
        # L679-L681: with every request 24 steps long the throughput bound is
        # bmax / (24 x t_step(bmax)); t_step measured here on full 512-row tasks, back to back
        rng = np.random.default_rng(5)
        b = 512
        slots = rng.choice(1 << 16, size=b, replace=False).astype(np.int32)
        rows = np.stack([rng.integers(3, WL[wl]["vocab"], size=b), np.zeros(b), slots,
                         (np.arange(b) % 2) * bm.ROW_PARITY], 1)
        cid = cells[gen.CHAIN][0]
        for _ in range(5):
            e.cell_step(cid, rows, sync=False)
        torch.cuda.synchronize()
        ev0.record(stream)
        for _ in range(50):
            e.cell_step(cid, rows, sync=False)
        ev1.record(stream)
        ev1.synchronize()
        t_step = ev0.elapsed_time(ev1) / 50 / 1e3
        b_req = b / (24 * t_step) * world
        bound = {"t_step_b512_us": t_step * 1e6, "bound_req_s": b_req, "fraction_of_bound": value / b_req,
                 "paper": "BatchMaker at ~87% of 27,136 req/s on V100 (L679-L681)"}
    if wl == "tree" and LENGTHS == "identical":
        # Fig. 15 (L857): identical complete 16-leaf trees against a hard-coded ideal that packs
        # every level of 64/16 = 4 trees into full tasks: per tree 16 leaf rows + 15 internal
        # rows, i.e. 16/64 of a 64-row leaf task + 15/64 of a 64-row internal task
        rng = np.random.default_rng(5)
        b = 64
        slots = rng.choice(1 << 16, size=3 * b, replace=False).astype(np.int32)
        leaf_rows = np.stack([rng.integers(3, WL[wl]["vocab"], size=b), np.zeros(b), slots[:b], np.zeros(b)], 1)
        int_rows = np.stack([slots[b:2 * b], slots[2 * b:], slots[:b], np.zeros(b)], 1)
        lf, it = cells[gen.TREE]
        t = {}
        for name, cid, rows in (("leaf", lf, leaf_rows), ("internal", it, int_rows)):
            for _ in range(5):
                e.cell_step(cid, rows, sync=False)
            torch.cuda.synchronize()
            ev0.record(stream)
            for _ in range(50):
                e.cell_step(cid, rows, sync=False)
            ev1.record(stream)
            ev1.synchronize()
            t[name] = ev0.elapsed_time(ev1) / 50 / 1e3
        ideal = world / (16 / b * t["leaf"] + 15 / b * t["internal"])
        bound = {"t_leaf_b64_us": t["leaf"] * 1e6, "t_internal_b64_us": t["internal"] * 1e6,
                 "ideal_req_s": ideal, "fraction_of_ideal": value / ideal,
                 "paper": "BatchMaker peak ~30% below the hard-coded ideal (L857)"}
    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_oracle(wl, a.cpu_seconds)
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "requests/sec", "n_gpus": world, "steps": a.steps,
                "warmup": a.warmup, "ms_per_step": t_max * 1e3 / a.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
                "config": {"workload": WL[wl]["config"] if LENGTHS == "wmt" else
                           (WL[wl]["config"].replace("WMT-like lengths", f"Fig. 11 lengths '{LENGTHS}'")
                            if wl == "lstm" else WL[wl]["config"] + "; identical complete 16-leaf trees (Fig. 15)"),
                           "requests_per_step": n_req,
                           "offered_rate_per_gpu": lam_star, "p90_bound_ms": bound_ms,
                           "p90_bound_kind": bound_kind,
                           "max_offered_rate_under": bounds if a.rate <= 0 else None,
                           "saturation_burst_rate_per_gpu": mu, "lookahead_k": a.lookahead,
                           "l2": "256 MB buffer written between timed steps; weights L2-resident within a "
                                 "step (serving)", "parallelism": f"request-sharded x{world}",
                           "persistent_kernel": bool(a.persistent), "workers_per_gpu": a.workers,
                           "bmax": ({"encoder": ENC_BMAX, "decoder": 256} if wl == "seq2seq" else
                                    (512 if wl == "lstm" else 64)),
                           "policy": ("cellular batching (Algorithm 1)" if policy == bm.POLICY_CELLULAR else
                                      f"graph-batching baseline: padding + bucketing, width {a.bucket_width}, "
                                      "round robin over buckets (L427)")},
                "latency_ms": {"p50": p50 * 1e3, "p90": p90 * 1e3, "p99": p99 * 1e3},
                # Fig. 9's decomposition (L597): queueing = arrival -> first node scheduled,
                # computation = first node -> completion
                "latency_split_ms": {k: dict(zip(("p50", "p90", "p99"), (x * 1e3 for x in shard.percentiles(v))))
                                     for k, v in (("queueing", q_lat), ("computation", c_lat))},
                "curve": curve, "e2e": e2e, "roofline": roof, "cpu_baseline": cpu, "analytic_bound": bound,
                "clocks": clk.summary(), "gpu_launches": int(st["kernel_launches"]),
                "sched_ns_per_task": st["sched_ns"] / max(1, st["tasks"])}
        s = json.dumps(line)
        print(s, flush=True)
        if a.out:
            with open(a.out, "w") as f:
                f.write(s + "\n")
    e.close()
    e2.close()
    if dist is not None:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
