"""End-to-end parity on the GPU (-m gpu): whole traces through the C-ABI engine (scheduler +
kernels), checked two ways (north_star):
  1. the scheduler's task log (batch composition, slot indices) and per-request completion
     order are bit-exact with the Python replay of Algorithm 1 (virtual clock, P9);
  2. every request's final h/c (and Seq2Seq tokens/logits) agree with the fp64 oracle run
     unbatched, within 5e-3 (bf16) / 1e-5 (fp32)."""
import numpy as np
import pytest

from oracle import batched, cells
from oracle.scheduler import CHAIN, SEQ2SEQ, TREE, Replay
from paper_conf_eurosys_gaoywl18_b200 import bm
from gpu_helpers import TOL, lstm_engine, seq2seq_engine, tree_engine
from workloads import gen

pytestmark = pytest.mark.gpu


def _check_log(e, rp):
    log = e.read_log()
    assert len(log) == len(rp.tasks)
    for a, t in zip(log, rp.tasks):
        assert a["cell"] == t.ct and a["tick"] == t.tick
        assert a["rows"] == [(r.rid, r.node, r.slot) for r in t.rows]
    comp = e.poll()
    assert [(c.req_id, c.t_done) for c in comp] == [(rid, float(tk)) for rid, tk in rp.completions]


@pytest.mark.parametrize("persistent", [0, 1])
@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
@pytest.mark.parametrize("minf", [1, 4])
def test_config0_end_to_end(prec, minf, persistent):
    """BASELINE configs[0]: 1-layer LSTM, h=64, 4 requests (3, 10, 5, 8), arrivals (0, 0, 1, 3),
    bmax 4, virtual clock; also through the persistent weight-stationary kernel (bf16)."""
    trace = gen.config0_trace(vocab=128)
    e, cid, w = lstm_engine(64, 1, 128, prec, bmax=4, clock=bm.CLOCK_VIRTUAL, max_slots=16,
                            max_requests=16, keep_results=1, min_followon_batch=minf,
                            persistent=persistent)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    e.run()
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    _check_log(e, Replay([(4, 0)], max_slots=16, min_followon=minf).run(reqs))
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, q.tokens)
        assert np.max(np.abs(r["h"][0] - hs[0])) <= TOL[prec]
        assert np.max(np.abs(r["c"][0] - cs[0])) <= TOL[prec]


@pytest.mark.parametrize("prec,persistent", [(bm.PREC_BF16, 0), (bm.PREC_BF16, 1), (bm.PREC_FP32, 0)])
def test_wmt_chain_h1024(prec, persistent):
    """configs[1] shape at a size the oracle finishes in seconds: 48 WMT-length requests,
    Poisson arrivals, h=1024, bmax 512, virtual clock with look-ahead k=2; bf16 also through the
    persistent weight-stationary kernel."""
    trace = gen.chain_trace(48, 2048, seed=1000, rate=2.0)
    e, cid, w = lstm_engine(1024, 1, 2048, prec, bmax=512, clock=bm.CLOCK_VIRTUAL, max_slots=256,
                            max_requests=256, keep_results=1, schedule_when_outstanding_leq=2,
                            persistent=persistent)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    e.run()
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    _check_log(e, Replay([(512, 0)], max_slots=256, schedule_when_outstanding_leq=2).run(reqs))
    worst = 0.0
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, q.tokens)
        worst = max(worst, np.max(np.abs(r["h"][0] - hs[0])), np.max(np.abs(r["c"][0] - cs[0])))
    assert worst <= TOL[prec], worst


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
@pytest.mark.parametrize("h,V,n", [(64, 256, 12), (1024, 32768, 6)])
def test_seq2seq_forced_tokens(prec, h, V, n):
    """Seq2Seq 4+4 layers, greedy feed-previous decoding on device. The oracle follows the GPU's
    emitted tokens (forced-token mode) and asserts each was a valid argmax within tolerance;
    then final h/c per layer and every step's logits are compared."""
    L = 4
    rng = np.random.default_rng(h)
    e, (ce, cd), (enc, dec) = seq2seq_engine(h, L, V, prec, bmax=(512, 256), clock=bm.CLOCK_VIRTUAL,
                                             max_slots=64, max_requests=64, keep_results=1,
                                             record_logits=1, max_decode_len=40)
    trace = []
    for i in range(n):
        S = int(rng.integers(1, 12))
        T = int(rng.integers(1, 12))
        trace.append((rng.integers(3, V, size=S).astype(np.int32), T, float(rng.integers(0, 6))))
    trace.sort(key=lambda x: x[2])
    for toks, T, t in trace:
        e.submit(bm.REQ_SEQ2SEQ, ce, cd, toks, t, decode_len=T)
    e.run()
    reqs = [{"kind": SEQ2SEQ, "cells": [0, 1], "arrival": t, "length": len(toks), "decode_len": T}
            for toks, T, t in trace]
    _check_log(e, Replay([(512, 0), (256, 1)], max_slots=64).run(reqs))
    tol = TOL[prec]
    for i, (toks, T, _) in enumerate(trace):
        r = e.read_result(i, L, decode_len=T, vocab=V)
        o = cells.seq2seq(enc, dec, toks, T, forced_tokens=r["tokens"])
        for s in range(T):
            assert o["logits"][s][r["tokens"][s]] >= o["logits"][s].max() - 2 * tol
        assert np.max(np.abs(r["logits"] - o["logits"])) <= tol
        for l in range(L):
            assert np.max(np.abs(r["h"][l] - o["h"][l])) <= tol
            assert np.max(np.abs(r["c"][l] - o["c"][l])) <= tol


def _s2s_trace(V, n, seed):
    rng = np.random.default_rng(seed)
    trace = []
    for i in range(n):
        S = int(rng.integers(1, 12))
        T = int(rng.integers(4, 14))
        trace.append((rng.integers(3, V, size=S).astype(np.int32), T, float(rng.integers(0, 6))))
    trace.sort(key=lambda x: x[2])
    return trace


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
@pytest.mark.parametrize("h,V,n", [(64, 256, 12), (1024, 32768, 6)])
def test_seq2seq_eos_terminated(prec, h, V, n):
    """§8f N1 (L715): decoding stops at <eos> or at the maximum length. The <eos> symbol is the
    token request 0 emits at some step j >= 1 in a fixed-length run, so at least one request
    terminates early (with V = 256 others do too). Checked: tokens after each request's <eos>
    are -1; the task log and completions are bit-exact with the replay given the <eos> steps
    the device produced (the replay learns each at the retire of its task, like the engine);
    the oracle in forced-token mode, stopping at the same <eos>, matches the emitted steps'
    logits and the final h/c of every layer (the state of the <eos> step: later, speculatively
    submitted steps were masked on the device)."""
    L = 4
    trace = _s2s_trace(V, n, h + 7)
    kw = dict(bmax=(512, 256), clock=bm.CLOCK_VIRTUAL, max_slots=64, max_requests=64, keep_results=1,
              record_logits=1, max_decode_len=40)
    e, (ce, cd), (enc, dec) = seq2seq_engine(h, L, V, prec, **kw)
    for toks, T, t in trace:
        e.submit(bm.REQ_SEQ2SEQ, ce, cd, toks, t, decode_len=T)
    e.run()
    y0 = e.read_result(0, L, decode_len=trace[0][1])["tokens"]
    j = next(i for i in range(1, len(y0)) if y0[i] not in y0[:i]) if len(set(y0)) > 1 else 0
    eos = int(y0[j])
    e.close()

    e, (ce, cd), (enc, dec) = seq2seq_engine(h, L, V, prec, **kw)
    for toks, T, t in trace:
        e.submit(bm.REQ_SEQ2SEQ, ce, cd, toks, t, decode_len=T, eos_id=eos)
    e.run()
    tol = TOL[prec]
    steps = []
    for i, (toks, T, _) in enumerate(trace):
        r = e.read_result(i, L, decode_len=T, vocab=V)
        y = [int(v) for v in r["tokens"]]
        m = y.index(-1) if -1 in y else T
        assert all(v == -1 for v in y[m:])
        assert all(v >= 0 for v in y[:m])
        if m < T:
            assert y[m - 1] == eos and eos not in y[:m - 1]
        steps.append(m - 1 if m < T or (m == T and y[T - 1] == eos) else None)
        o = cells.seq2seq(enc, dec, toks, T, forced_tokens=y[:m], eos_id=eos)
        assert len(o["tokens"]) == m
        for s in range(m):
            assert o["logits"][s][y[s]] >= o["logits"][s].max() - 2 * tol
        assert np.max(np.abs(r["logits"][:m] - o["logits"])) <= tol
        for l in range(L):
            assert np.max(np.abs(r["h"][l] - o["h"][l])) <= tol
            assert np.max(np.abs(r["c"][l] - o["c"][l])) <= tol
    assert steps[0] == j
    # the bulk read reports the same tokens, -1 after each request's last emitted one
    bulk = np.zeros((n, 40), np.int32)
    e.read_results_many(0, n, tokens=bulk, release=False)
    for i, (toks, T, _) in enumerate(trace):
        m = (steps[i] + 1) if steps[i] is not None else T
        one = e.read_result(i, L, decode_len=T)["tokens"]
        assert list(bulk[i, :T]) == list(one) and (bulk[i, m:] == -1).all()
    reqs = [{"kind": SEQ2SEQ, "cells": [0, 1], "arrival": t, "length": len(toks), "decode_len": T,
             "eos_step": steps[i]} for i, (toks, T, t) in enumerate(trace)]
    _check_log(e, Replay([(512, 0), (256, 1)], max_slots=64).run(reqs))
    e.close()


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
def test_treebank_trees_h1024(prec):
    """configs[3] shape: TreeBank-like binary trees + the identical complete 16-leaf tree,
    leaf and internal cell types batched separately (bmax 64), virtual clock."""
    V = 4096
    trace = gen.tree_trace(10, V, seed=3000, rate=1.0) + gen.tree_trace(2, V, seed=3001, identical=True)
    for j, q in enumerate(trace):
        q.arrival = float(j // 3)
    e, (leaf, intern), w = tree_engine(1024, V, prec, bmax=64, clock=bm.CLOCK_VIRTUAL, max_slots=1024,
                                       max_requests=64, keep_results=1)
    for q in trace:
        e.submit(bm.REQ_TREE, leaf, intern, q.tokens, q.arrival, left=q.left, right=q.right)
    e.run()
    reqs = [{"kind": TREE, "cells": [0, 1], "arrival": q.arrival, "left": q.left, "right": q.right}
            for q in trace]
    _check_log(e, Replay([(64, 0), (64, 1)], max_slots=1024).run(reqs))
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        rh, rc, _ = cells.tree_lstm(w, q.tokens, q.left, q.right)
        assert np.max(np.abs(r["h"][0] - rh)) <= TOL[prec]
        assert np.max(np.abs(r["c"][0] - rc)) <= TOL[prec]


@pytest.mark.parametrize("persistent", [0, 1])
def test_wall_clock_run_completes_and_matches_oracle(persistent):
    """The open-loop driver on the wall clock (bench path): all requests complete, results
    match the oracle (scheduling then depends on timing, results must not)."""
    trace = gen.chain_trace(64, 1024, seed=5, rate=20000.0)
    e, cid, w = lstm_engine(1024, 1, 1024, bm.PREC_BF16, bmax=512, max_slots=256, max_requests=256,
                            keep_results=1, schedule_when_outstanding_leq=2, persistent=persistent)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    assert e.run() == 64
    comp = e.poll()
    assert sorted(c.req_id for c in comp) == list(range(64))
    for i in (0, 17, 63):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, trace[i].tokens)
        assert np.max(np.abs(r["h"][0] - hs[0])) <= TOL[bm.PREC_BF16]
    # a second run on the same engine (the persistent kernel is relaunched per bm_run)
    for q in trace[:8]:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    assert e.run() == 8


def test_persistent_large_batches_match_launch_path():
    """Persistent kernel with 300-row tasks (3 column chunks) equals the per-task launch path
    on the same trace (both bf16, results within tolerance of each other and the oracle)."""
    trace = gen.chain_trace(600, 1024, seed=9, lengths=[3] * 600, arrivals=[0] * 600)
    res = []
    for persistent in (0, 1):
        e, cid, w = lstm_engine(1024, 1, 1024, bm.PREC_BF16, bmax=300, clock=bm.CLOCK_VIRTUAL,
                                max_slots=1024, max_requests=1024, keep_results=1, persistent=persistent)
        for q in trace:
            e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
        assert e.run() == 600
        res.append(np.stack([e.read_result(i, 1)["h"][0] for i in range(600)]))
    # every request of both paths against the fp64 oracle (batched executor, pinned by P4)
    toks = [q.tokens for q in trace]
    ref = batched.run_chain_schedule(w, toks, [[(r, k) for r in range(600)] for k in range(3)])
    for p in (0, 1):
        err = max(np.max(np.abs(res[p][i] - ref[i][0][0])) for i in range(600))
        assert err <= TOL[bm.PREC_BF16], (p, err)


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
def test_graph_batching_policy_h1024(prec):
    """N4: the padding + bucketing baseline (§7.1) on the same kernels -- task log and
    completions bit-exact with its replay, and padding does not change any request's result
    (the result row is the real last step; padded steps run on the pad token afterwards)."""
    from oracle.scheduler import GraphBatchingReplay
    trace = gen.chain_trace(40, 2048, seed=1001, rate=1.0)
    e, cid, w = lstm_engine(1024, 1, 2048, prec, bmax=16, clock=bm.CLOCK_VIRTUAL, max_slots=256,
                            max_requests=256, keep_results=1, schedule_when_outstanding_leq=1,
                            policy=bm.POLICY_GRAPH, bucket_width=10)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    assert e.run() == len(trace)
    rp = GraphBatchingReplay(16, max_slots=256, bucket_width=10, schedule_when_outstanding_leq=1)
    rp.run([dict(arrival=q.arrival, length=q.length) for q in trace])
    log = e.read_log()
    assert len(log) == len(rp.tasks)
    for a, t in zip(log, rp.tasks):
        assert a["tick"] == t.tick and a["rows"] == [(r.rid, r.node, r.slot) for r in t.rows]
    comp = e.poll()
    assert [(c.req_id, c.t_done) for c in comp] == [(rid, float(tk)) for rid, tk in rp.completions]
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, q.tokens)
        assert np.max(np.abs(r["h"][0] - hs[0])) <= TOL[prec]
        assert np.max(np.abs(r["c"][0] - cs[0])) <= TOL[prec]


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
def test_two_workers_chain_h1024(prec):
    """§8f N2 on one device: two Algorithm-1 workers (two streams, subgraphs pinned to the worker
    running them, L317/L381). Virtual clock: the task log (worker included) equals the replay
    with W = 2; every request's final state matches the oracle."""
    trace = gen.chain_trace(48, 2048, seed=1001, rate=3.0)
    e, cid, w = lstm_engine(1024, 1, 2048, prec, bmax=512, clock=bm.CLOCK_VIRTUAL, max_slots=256,
                            max_requests=256, keep_results=1, schedule_when_outstanding_leq=2, workers=2)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    e.run()
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    rp = Replay([(512, 0)], max_slots=256, schedule_when_outstanding_leq=2, workers=2).run(reqs)
    assert {t.worker for t in rp.tasks} == {0, 1}
    _check_log(e, rp)
    worst = 0.0
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, q.tokens)
        worst = max(worst, np.max(np.abs(r["h"][0] - hs[0])), np.max(np.abs(r["c"][0] - cs[0])))
    assert worst <= TOL[prec], worst


def test_two_workers_seq2seq_eos():
    """Two workers with the Seq2Seq decoder (projection scratch per worker) and <eos> stop."""
    h, V, L = 64, 256, 4
    trace = _s2s_trace(V, 12, 99)
    kw = dict(bmax=(512, 256), clock=bm.CLOCK_VIRTUAL, max_slots=64, max_requests=64, keep_results=1,
              max_decode_len=40, workers=2)
    e, (ce, cd), (enc, dec) = seq2seq_engine(h, L, V, bm.PREC_BF16, **kw)
    eos = 7
    for toks, T, t in trace:
        e.submit(bm.REQ_SEQ2SEQ, ce, cd, toks, t, decode_len=T, eos_id=eos)
    e.run()
    steps = []
    for i, (toks, T, _) in enumerate(trace):
        r = e.read_result(i, L, decode_len=T)
        y = [int(v) for v in r["tokens"]]
        m = y.index(-1) if -1 in y else T
        steps.append(m - 1 if (m < T or y[T - 1] == eos) else None)
        o = cells.seq2seq(enc, dec, toks, T, forced_tokens=y[:m], eos_id=eos)
        for l in range(L):
            assert np.max(np.abs(r["h"][l] - o["h"][l])) <= TOL[bm.PREC_BF16]
    reqs = [{"kind": SEQ2SEQ, "cells": [0, 1], "arrival": t, "length": len(toks), "decode_len": T,
             "eos_step": steps[i]} for i, (toks, T, t) in enumerate(trace)]
    _check_log(e, Replay([(512, 0), (256, 1)], max_slots=64, workers=2).run(reqs))


def test_two_workers_wall_clock():
    """Two workers on the wall clock (the bench path): all requests complete, sampled results
    match the oracle."""
    trace = gen.chain_trace(400, 1024, seed=6, rate=200000.0)
    e, cid, w = lstm_engine(1024, 1, 1024, bm.PREC_BF16, bmax=512, max_slots=1024, max_requests=1024,
                            keep_results=1, schedule_when_outstanding_leq=2, workers=2)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    assert e.run() == 400
    assert sorted(c.req_id for c in e.poll()) == list(range(400))
    for i in (0, 123, 399):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, trace[i].tokens)
        assert np.max(np.abs(r["h"][0] - hs[0])) <= TOL[bm.PREC_BF16]


def _wmt_replay_case(n=40, k=2):
    trace = gen.chain_trace(n, 2048, seed=1001, rate=2.0)
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    rp = Replay([(512, 0)], max_slots=256, schedule_when_outstanding_leq=k).run(reqs)
    return trace, rp


def _check_log_only(e, rp):
    log = e.read_log()
    assert len(log) == len(rp.tasks)
    for a, t in zip(log, rp.tasks):
        assert a["cell"] == t.ct and a["tick"] == t.tick
        assert a["rows"] == [(r.rid, r.node, r.slot) for r in t.rows]


def test_schedule_step_and_poll_by_hand():
    """The paper's boundary driven call by call (no bm_run): bm_schedule_step (retire, admit,
    Schedule when idle, launch; the virtual clock advances to the next event) until BM_E_AGAIN,
    with bm_poll after every step. The task log, slots and the completions bm_poll returned, in
    order, equal the Algorithm-1 replay; every result equals the fp64 oracle."""
    trace, rp = _wmt_replay_case()
    e, cid, w = lstm_engine(1024, 1, 2048, bm.PREC_BF16, bmax=512, clock=bm.CLOCK_VIRTUAL, max_slots=256,
                            max_requests=256, keep_results=1, schedule_when_outstanding_leq=2)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    comps = []
    for _ in range(100000):
        n = e.schedule_step()
        comps += e.poll()
        if n < 0:
            break
    assert n < 0
    _check_log_only(e, rp)
    assert [(c.req_id, c.t_done) for c in comps] == [(rid, float(tk)) for rid, tk in rp.completions]
    worst = 0.0
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, q.tokens)
        worst = max(worst, np.max(np.abs(r["h"][0] - hs[0])), np.max(np.abs(r["c"][0] - cs[0])))
    assert worst <= TOL[bm.PREC_BF16], worst
    e.close()


@pytest.mark.parametrize("driver", ["schedule_step", "run"])
def test_poll_thread_concurrent(driver):
    """bm_poll on its own thread (the paper's polling thread, L395) while the main thread drives
    the engine (bm_schedule_step loop, or bm_run): the engine lock serialises them, so the task
    log and the completion order the poll thread sees are bit-exact with the replay."""
    import threading
    trace, rp = _wmt_replay_case(n=48)
    e, cid, w = lstm_engine(1024, 1, 2048, bm.PREC_BF16, bmax=512, clock=bm.CLOCK_VIRTUAL, max_slots=256,
                            max_requests=256, keep_results=1, schedule_when_outstanding_leq=2)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    got, stop = [], threading.Event()

    def poller():
        while not stop.is_set() or len(got) < len(trace):
            got.extend(e.poll(64))
            if stop.is_set() and len(got) >= len(trace):
                break

    th = threading.Thread(target=poller)
    th.start()
    if driver == "run":
        assert e.run() == len(trace)
    else:
        while e.schedule_step() >= 0:
            pass
    stop.set()
    th.join(timeout=60)
    assert not th.is_alive()
    _check_log_only(e, rp)
    assert [(c.req_id, c.t_done) for c in got] == [(rid, float(tk)) for rid, tk in rp.completions]
    e.close()


def test_weights_adopted_from_device_pointers():
    """bm_load_cell with DEVICE pointers (fp32 CUDA tensors, as after the NCCL broadcast of
    bench.py / shard.py): the weights are packed in place, no host round trip; a step then
    matches the same engine loaded from host arrays bit for bit."""
    import torch
    h, V, b = 1024, 512, 64
    w = gen.lstm_stack_weights(h, 1, V, 3)
    rng = np.random.default_rng(3)
    rows = np.stack([rng.integers(3, V, size=b), np.zeros(b), np.arange(b), bm.ROW_LAST | bm.ROW_FIRST |
                     (np.arange(b) << 8)], 1).astype(np.int32)
    out = []
    for dev in (False, True):
        e = bm.Engine(hidden=h, pool_layers=1, max_slots=256, max_requests=256)
        if dev:
            t = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.float32)).cuda()
            cid = e.load_cell(bm.CELL_LSTM, 1, V, 512, 0, [t(w.W[0])], [t(w.b[0])], t(w.E))
        else:
            cid = e.load_cell(bm.CELL_LSTM, 1, V, 512, 0, w.W, w.b, w.E)
        e.cell_step(cid, rows)
        out.append(e.result_rows(np.arange(b)))
        e.close()
    np.testing.assert_array_equal(out[0][0], out[1][0])
    np.testing.assert_array_equal(out[0][1], out[1][1])
    hs, cs = cells.lstm_cell(w.W[0], w.b[0], w.E[rows[0, 0]], np.zeros(h), np.zeros(h))
    assert np.max(np.abs(out[1][0][0, 0] - hs)) <= 2e-4


def test_two_devices_chain_and_trees_h1024():
    """§8f N2 across GPUs, functional on one B200: two workers on two DEVICE CONTEXTS (each with
    its own weight replica and state pool; on a multi-GPU box they are two GPUs). A subgraph
    scheduled on the other context carries its state rows along (peer copies, L337). The task
    log equals the replay worker for worker, the moves equal the replay's count (> 0), and every
    request's result equals the oracle -- wrong or missing migrations would corrupt them."""
    # sparse arrivals: a chain subgraph is pinned while a task of it is in flight (L381), so it
    # only changes worker when it goes idle between tasks; at rate 0.3 that happens (4 moves)
    trace = gen.chain_trace(48, 2048, seed=1003, rate=0.3)
    e, cid, w = lstm_engine(1024, 1, 2048, bm.PREC_BF16, bmax=64, clock=bm.CLOCK_VIRTUAL, max_slots=256,
                            max_requests=256, keep_results=1, max_tasks_to_submit=1, workers=2, devices=2)
    for q in trace:
        e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
    e.run()
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    rp = Replay([(64, 0)], max_slots=256, max_tasks_to_submit=1, workers=2, devices=2).run(reqs)
    _check_log(e, rp)
    assert e.stats()["migrations"] == rp.migrations > 0
    worst = 0.0
    for i, q in enumerate(trace):
        r = e.read_result(i, 1)
        hs, cs = cells.chain_lstm(w, q.tokens)
        worst = max(worst, np.max(np.abs(r["h"][0] - hs[0])), np.max(np.abs(r["c"][0] - cs[0])))
    assert worst <= TOL[bm.PREC_BF16], worst
    e.close()
    # trees: leaves and internal levels spread over the two contexts
    tt = gen.tree_trace(24, 1000, seed=8, rate=2.0)
    e, (leaf, intern), tw = tree_engine(1024, 1000, bm.PREC_BF16, bmax=16, clock=bm.CLOCK_VIRTUAL, max_slots=2048,
                                        max_requests=64, keep_results=1, max_tasks_to_submit=1, workers=2, devices=2)
    for q in tt:
        e.submit(bm.REQ_TREE, leaf, intern, q.tokens, q.arrival, left=q.left, right=q.right)
    e.run()
    rq = [{"kind": TREE, "cells": [0, 1], "arrival": q.arrival, "left": q.left, "right": q.right} for q in tt]
    rp = Replay([(16, 0), (16, 1)], max_slots=2048, max_tasks_to_submit=1, workers=2, devices=2).run(rq)
    _check_log(e, rp)
    assert e.stats()["migrations"] == rp.migrations > 0
    for i, q in enumerate(tt):
        r = e.read_result(i, 1)
        rh, rc, _ = cells.tree_lstm(tw, q.tokens, q.left, q.right)
        assert np.max(np.abs(r["h"][0] - rh)) <= TOL[bm.PREC_BF16] and np.max(np.abs(r["c"][0] - rc)) <= TOL[bm.PREC_BF16]


def test_two_devices_seq2seq_eos():
    """Two device contexts with the Seq2Seq decoder: the feed token and the <eos> mark move with
    the request's state rows (greedy feed-previous stays on the token the device emitted)."""
    h, V, L = 64, 256, 4
    trace = _s2s_trace(V, 12, 98)
    kw = dict(bmax=(4, 4), clock=bm.CLOCK_VIRTUAL, max_slots=64, max_requests=64, keep_results=1,
              max_decode_len=40, workers=2, devices=2, max_tasks_to_submit=1)
    e, (ce, cd), (enc, dec) = seq2seq_engine(h, L, V, bm.PREC_BF16, **kw)
    eos = 7
    for toks, T, t in trace:
        e.submit(bm.REQ_SEQ2SEQ, ce, cd, toks, t, decode_len=T, eos_id=eos)
    e.run()
    steps = []
    for i, (toks, T, _) in enumerate(trace):
        r = e.read_result(i, L, decode_len=T)
        y = [int(v) for v in r["tokens"]]
        m = y.index(-1) if -1 in y else T
        steps.append(m - 1 if (m < T or y[T - 1] == eos) else None)
        o = cells.seq2seq(enc, dec, toks, T, forced_tokens=y[:m], eos_id=eos)
        for s in range(m):
            assert o["logits"][s][y[s]] >= o["logits"][s].max() - 2 * TOL[bm.PREC_BF16]
        for l in range(L):
            assert np.max(np.abs(r["h"][l] - o["h"][l])) <= TOL[bm.PREC_BF16]
    reqs = [{"kind": SEQ2SEQ, "cells": [0, 1], "arrival": t, "length": len(toks), "decode_len": T,
             "eos_step": steps[i]} for i, (toks, T, t) in enumerate(trace)]
    rp = Replay([(4, 0), (4, 1)], max_slots=64, workers=2, devices=2, max_tasks_to_submit=1).run(reqs)
    _check_log(e, rp)
    assert e.stats()["migrations"] == rp.migrations > 0
