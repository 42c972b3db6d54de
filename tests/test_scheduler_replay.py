"""Pins for the scheduler replay oracle: Algorithm 1 (L345-L369) with the
request processor (L323, L341, L383-L385), checked against the paper's printed Figure 5
schedule, the §4.4 TreeLSTM walk-through, and invariants that any correct cellular
batching scheduler must satisfy (hypothesis)."""
import json
import os

import numpy as np
import pytest
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

from oracle.scheduler import CHAIN, SEQ2SEQ, TREE, Replay, replay_requests
from workloads import gen

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _run_chain(trace, bmax, min_followon, max_tasks=5, k=0, max_slots=1 << 20):
    return replay_requests(trace, {CHAIN: [0]}, cell_types=[(bmax, 0)],
                           max_tasks_to_submit=max_tasks, min_followon=min_followon,
                           schedule_when_outstanding_leq=k, max_slots=max_slots)


# ----------------------------------------------------------------------------- P5 Figure 5
def test_p5_figure5_printed_tasks():
    g = json.load(open(os.path.join(GOLD, "figure5.json")))
    trace = gen.figure5_trace()
    assert [q.length for q in trace] == g["lengths"]
    assert [q.arrival for q in trace] == g["unprinted_arrivals_reading"]["arrivals"]
    # Graph batching numbers printed in the same figure follow from the lengths alone.
    assert max(g["lengths"][:4]) == g["printed_graph_batching"]["batch1_end"]
    assert (max(g["lengths"][:4]) + max(g["lengths"][4:])
            == g["printed_graph_batching"]["batch2_end"])
    rp = _run_chain(trace, g["batch_size"], min_followon=g["batch_size"])
    members = [sorted(r.rid + 1 for r in t.rows) for t in rp.tasks[:4]]
    assert members == g["printed_cellular_tasks"]["tasks_1_to_4_members"]
    assert rp.tasks[2].tick == g["printed_cellular_tasks"]["task3_start_tick"]
    assert rp.reqs[0].complete_tick == g["printed_cellular_tasks"]["req1_completes_tick"]


def test_p5_figure5_full_schedule_min4():
    """Whole schedule under the arrival reading (computed independently there):
    ticks 0-9 {1-4},{1-4},{2-5},{4-7},{4-7},{5-8},{5,6},{6},{6},{6};
    completion ticks req1..8 = 2,3,3,5,7,10,6,6."""
    rp = _run_chain(gen.figure5_trace(), 4, 4)
    got = [(t.tick, sorted(r.rid + 1 for r in t.rows)) for t in rp.tasks]
    assert got == [(0, [1, 2, 3, 4]), (0, [1, 2, 3, 4]), (2, [2, 3, 4, 5]), (2, [4, 5, 6, 7]),
                   (2, [4, 5, 6, 7]), (5, [5, 6, 7, 8]), (6, [5, 6]), (7, [6]), (8, [6]), (9, [6])]
    assert [rp.reqs[i].complete_tick for i in range(8)] == [2, 3, 3, 5, 7, 10, 6, 6]


def test_p5_figure5_min1_differs():
    """With Bsizes.Min() = 1 the third task is {2,3,4} at t=0 (line 16 submits it), so the
    printed figure requires Min = bmax (reading S14)."""
    rp = _run_chain(gen.figure5_trace(), 4, 1)
    assert sorted(r.rid + 1 for r in rp.tasks[2].rows) == [2, 3, 4]
    assert rp.tasks[2].tick == 0


@pytest.mark.parametrize("min_followon,n_tasks,complete", [(1, 13, [3, 10, 10, 13]),
                                                           (4, 11, [3, 10, 6, 11])])
def test_config0_fixture(min_followon, n_tasks, complete):
    """BASELINE configs[0] trace: expectations derived there."""
    rp = _run_chain(gen.config0_trace(), 4, min_followon)
    assert len(rp.tasks) == n_tasks
    assert [r.complete_tick for r in rp.reqs] == complete


# ----------------------------------------------------------------------------- P6 §4.4
def test_p6_complete_tree_walkthrough():
    """§4.4: a complete binary tree with 16 leaves -> 17 subgraphs (16 single-leaf
    + 1 internal); leaves queued at once, the internal subgraph only after every leaf
    finished; successive levels in successive tasks (reading S12: 15 internal nodes)."""
    left, right = gen.complete_tree(16)
    rp = Replay([(64, 0), (64, 1)], max_tasks_to_submit=5)
    rp.run([{"kind": TREE, "cells": [0, 1], "arrival": 0, "left": left, "right": right}])
    r = rp.reqs[0]
    assert len(r.subgraphs) == 17
    assert sum(len(sg.nodes) == 1 for sg in r.subgraphs) == 16
    assert len(r.subgraphs[-1].nodes) == 15
    sizes = [(t.ct, len(t.rows), t.tick) for t in rp.tasks]
    assert sizes == [(0, 16, 0), (1, 8, 1), (1, 4, 1), (1, 2, 1), (1, 1, 1)]
    # task k of the internal subgraph holds exactly the height-k nodes
    for k, t in enumerate(rp.tasks[1:], start=1):
        assert all(r.height[row.node] == k for row in t.rows)
    assert r.complete_tick == 5


def test_seq2seq_decoder_released_at_encoder_completion():
    rp = Replay([(8, 0), (8, 1)], max_tasks_to_submit=5)
    rp.run([{"kind": SEQ2SEQ, "cells": [0, 1], "arrival": 0, "length": 3, "decode_len": 2}])
    assert [(t.ct, t.tick) for t in rp.tasks] == [(0, 0), (0, 0), (0, 0), (1, 3), (1, 3)]
    assert rp.reqs[0].complete_tick == 5


def test_priority_decoder_over_encoder():
    """L339: later cells first — with both types ready and running, the higher priority
    (decoder) wins tier (c)."""
    rp = Replay([(8, 0), (8, 1)], max_tasks_to_submit=1)
    rp.run([{"kind": SEQ2SEQ, "cells": [0, 1], "arrival": 0, "length": 1, "decode_len": 3},
            {"kind": SEQ2SEQ, "cells": [0, 1], "arrival": 1, "length": 4, "decode_len": 1}])
    # at tick 1: req0 decoder ready (priority 1) and req1 encoder ready -> decoder first
    assert rp.tasks[1].ct == 1


def test_slot_exhaustion_defers_and_reuses_lowest_slot():
    trace = gen.chain_trace(3, 16, 0, lengths=[2, 2, 2], arrivals=[0, 0, 0])
    rp = _run_chain(trace, 4, 1, max_slots=2)
    first = rp.tasks[0]
    assert [r.slot for r in first.rows] == [0, 1]
    later = [t for t in rp.tasks if any(r.rid == 2 for r in t.rows)]
    assert later[0].rows[0].slot == 0            # lowest freed slot reused
    assert all(r.complete_tick is not None for r in rp.reqs)


# ----------------------------------------------------------------------------- P7 invariants
def check_invariants(rp: Replay, reqs):
    cts = rp.cts
    node_task = {}
    for t in rp.tasks:
        assert 0 < len(t.rows) <= cts[t.ct].bmax
        slots = [r.slot for r in t.rows]
        assert len(set(slots)) == len(slots), "slot twice in one task"
        for row in t.rows:
            key = (row.rid, row.node)
            assert key not in node_task, "node ran twice"
            node_task[key] = t
    for r in rp.reqs:
        q = reqs[r.rid]
        assert all((r.rid, v) in node_task for v in range(r.n_nodes)), "node never ran"
        last_finish = max(node_task[(r.rid, v)].finish for v in range(r.n_nodes))
        assert r.complete_tick == last_finish, "completion not at last node's retire"
        for v in range(r.n_nodes):
            t = node_task[(r.rid, v)]
            assert t.tick >= q["arrival"]
            if r.kind in (CHAIN, SEQ2SEQ) and v > 0:
                assert node_task[(r.rid, v - 1)].index < t.index
            if r.kind == SEQ2SEQ and v == r.enc_len and v > 0:
                assert t.tick >= node_task[(r.rid, v - 1)].finish, "decoder before encoder done"
            if r.kind == TREE and r.left[v] >= 0:
                for ch in (r.left[v], r.right[v]):
                    assert node_task[(r.rid, ch)].index < t.index
                leaves = [u for u in range(r.n_nodes) if r.left[u] < 0]
                assert t.tick >= max(node_task[(r.rid, u)].finish for u in leaves)
    # no slot is held by two live requests at once
    spans = {}
    for r in rp.reqs:
        for s in set(r.slots.values()):
            spans.setdefault(s, []).append((r.first_tick, r.complete_tick))
    for s, iv in spans.items():
        iv.sort()
        for a, b in zip(iv, iv[1:]):
            assert b[0] >= a[1], f"slot {s} shared by live requests"
    for ct in cts:
        assert ct.running_tasks == 0 and not ct.queue
    for r in rp.reqs:
        for sg in r.subgraphs:
            assert sg.inflight == 0 and sg.pinned is None
    assert sorted(rid for rid, _ in rp.completions) == list(range(len(rp.reqs)))


def _random_requests(draw_data, n, kinds, vocab=32):
    out = []
    rng = np.random.default_rng(draw_data["seed"])
    t = 0.0
    for i in range(n):
        t += float(rng.integers(0, 3))
        kind = kinds[int(rng.integers(0, len(kinds)))]
        if kind == CHAIN:
            out.append({"kind": CHAIN, "cells": [0], "arrival": t, "length": int(rng.integers(1, 9))})
        elif kind == SEQ2SEQ:
            out.append({"kind": SEQ2SEQ, "cells": [1, 2], "arrival": t,
                        "length": int(rng.integers(1, 6)), "decode_len": int(rng.integers(1, 6))})
        else:
            left, right = gen._random_bracketing(int(rng.integers(1, 9)), rng)
            out.append({"kind": TREE, "cells": [3, 4], "arrival": t, "left": left, "right": right})
    return out


@settings(max_examples=400, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 10_000), n=st.integers(1, 14),
       bmax=st.lists(st.integers(1, 6), min_size=5, max_size=5),
       prio=st.permutations([0, 1, 2, 3, 4]), max_tasks=st.integers(1, 5),
       min_followon=st.integers(1, 4), k=st.integers(0, 3), slots=st.integers(4, 40),
       kinds=st.sampled_from([[CHAIN], [SEQ2SEQ], [TREE], [CHAIN, SEQ2SEQ, TREE]]))
def test_p7_invariants_hypothesis(seed, n, bmax, prio, max_tasks, min_followon, k, slots, kinds):
    reqs = _random_requests({"seed": seed}, n, kinds)
    need = max((len(q["left"]) if q["kind"] == TREE else 1) for q in reqs)
    rp = Replay(list(zip(bmax, prio)), max_slots=max(slots, need),
                max_tasks_to_submit=max_tasks, min_followon=min_followon,
                schedule_when_outstanding_leq=k)
    rp.run(reqs)
    check_invariants(rp, reqs)


def test_p7_queueing_bound_under_light_load():
    """L629: an arriving request waits at most MaxTasksToSubmit steps when the system is
    not saturated (the in-flight look-ahead is the only wait)."""
    trace = gen.chain_trace(200, 64, 3, rate=0.05)
    rp = _run_chain(trace, 512, 1)
    for r, q in zip(rp.reqs, trace):
        assert r.first_tick - q.arrival <= 5 + 1e-9


def test_p7_fixed_length_throughput_bound():
    """L679-L681: with fixed length 24 the throughput cannot exceed bmax / (24 * t_step)."""
    trace = gen.chain_trace(600, 64, 4, lengths=[24] * 600, arrivals=[0] * 600)
    rp = _run_chain(trace, 64, 1)
    span = max(r.complete_tick for r in rp.reqs)
    assert len(trace) / span <= 64 / 24 + 1e-9


# ---------------------------------------------------------------- §8f N1: <eos>-terminated decode
def _s2s(length, T, eos_step, arrival=0.0):
    return {"kind": SEQ2SEQ, "cells": [0, 1], "arrival": arrival, "length": length, "decode_len": T,
            "eos_step": eos_step}


@pytest.mark.parametrize("eos_step,n_tasks,complete", [(1, 7, 7.0), (4, 7, 7.0), (None, 8, 8.0), (0, 7, 7.0)])
def test_n1_eos_hand_computed(eos_step, n_tasks, complete):
    """One request, 2 encoder steps, at most 6 decoder steps, bmax 4, MaxTasks 5, idle-only
    Schedule (k = 0), one tick per task. Tick 0: encoder tasks [e0] [e1] (successor ready at
    submit, L381); tick 2: the encoder completes -> the decoder subgraph is released (L331) and
    one Schedule call submits d0..d4 (MaxTasksToSubmit = 5, L379), finishing at ticks 3..7.
    The <eos> is learned at the retire of its task (d1: tick 4; d4: tick 7); d0..d4 are already
    in flight, so with <eos> at any step <= 4 nothing more is submitted and the request
    completes at tick 7 (7 tasks). Without <eos> d5 runs at tick 7 -> completion at 8 (L715)."""
    rp = Replay([(4, 0), (4, 1)]).run([_s2s(2, 6, eos_step)])
    assert len(rp.tasks) == n_tasks
    assert rp.completions == [(0, complete)]
    assert [t.rows[0].node for t in rp.tasks] == list(range(n_tasks))


@settings(max_examples=200, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 100_000), n=st.integers(1, 12), bmax=st.integers(1, 6),
       max_tasks=st.integers(1, 5), k=st.integers(0, 3))
def test_n1_eos_invariants(seed, n, bmax, max_tasks, k):
    """For every request with <eos> at decode step e: the decoder ran steps 0..m-1 with
    e < m <= T (nothing is skipped, the <eos> step ran, speculative steps are bounded by T); no
    decoder step was submitted after the retire of the task that emitted <eos> (the scheduler
    stops as soon as it learns of it); the request completes at the retire of its last
    submitted node; requests without <eos> run all T steps."""
    rng = np.random.default_rng(seed)
    reqs, t = [], 0.0
    for _ in range(n):
        t += float(rng.integers(0, 3))
        T = int(rng.integers(1, 9))
        e = int(rng.integers(0, T + 2))
        reqs.append(_s2s(int(rng.integers(1, 5)), T, e if e < T else None, t))
    rp = Replay([(bmax, 0), (bmax, 1)], max_tasks_to_submit=max_tasks,
                schedule_when_outstanding_leq=k).run(reqs)
    done = dict(rp.completions)
    for rid, q in enumerate(reqs):
        L = q["length"]
        dec = [(task, row.node - L) for task in rp.tasks for row in task.rows
               if row.rid == rid and row.node >= L]
        steps = sorted(s for _, s in dec)
        m = len(steps)
        assert steps == list(range(m))
        last_finish = max(task.finish for task in rp.tasks for row in task.rows if row.rid == rid)
        assert done[rid] == last_finish
        if q["eos_step"] is None:
            assert m == q["decode_len"]
        else:
            e = q["eos_step"]
            assert e < m <= q["decode_len"]
            t_eos = next(task.finish for task, s in dec if s == e)
            assert all(task.tick < t_eos for task, _ in dec)



# ---------------------------------------------------------------- §8f N2: several workers
@settings(max_examples=200, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 100_000), n=st.integers(1, 16), bmax=st.integers(1, 6),
       max_tasks=st.integers(1, 5), k=st.integers(0, 3), workers=st.integers(1, 4))
def test_n2_pinning_invariants(seed, n, bmax, max_tasks, k, workers):
    """Algorithm 1 with W workers (L345-L381): every node runs once; each worker runs its tasks
    one at a time; a subgraph never has nodes in flight on two workers at once (it is pinned to
    the worker that runs it until its in-flight count drops to 0, lines 21/27, L381); a task
    holds nodes of ready subgraphs only (dependencies as with one worker)."""
    rng = np.random.default_rng(seed)
    reqs, t = [], 0.0
    for _ in range(n):
        t += float(rng.integers(0, 3))
        if rng.random() < 0.5:
            reqs.append({"kind": CHAIN, "cells": [0], "arrival": t, "length": int(rng.integers(1, 9))})
        else:
            reqs.append({"kind": SEQ2SEQ, "cells": [0, 1], "arrival": t, "length": int(rng.integers(1, 5)),
                         "decode_len": int(rng.integers(1, 6))})
    rp = Replay([(bmax, 0), (bmax, 1)], max_tasks_to_submit=max_tasks, schedule_when_outstanding_leq=k,
                workers=workers).run(reqs)
    seen = set()
    for task in rp.tasks:
        for row in task.rows:
            assert (row.rid, row.node) not in seen
            seen.add((row.rid, row.node))
    assert len(seen) == sum(q["length"] + q.get("decode_len", 0) for q in reqs)
    for w in range(workers):
        mine = sorted((t_.tick, t_.finish) for t_ in rp.tasks if t_.worker == w)
        for (a0, a1), (b0, b1) in zip(mine, mine[1:]):
            assert b1 >= a1 + 1          # one task per tick per worker
    # pinning: intervals [tick, finish) of one subgraph's tasks on different workers are disjoint
    spans = {}
    for task in rp.tasks:
        for row in task.rows:
            r = rp.reqs[row.rid]
            sg = r.node_sg[row.node]
            spans.setdefault(id(sg), []).append((task.tick, task.finish, task.worker))
    for lst in spans.values():
        for i, (s0, f0, w0) in enumerate(lst):
            for s1, f1, w1 in lst[i + 1:]:
                if w0 != w1:
                    assert f0 <= s1 or f1 <= s0
    # a chain's steps run in order: step v+1's task is submitted no earlier than step v's
    for rid, r in enumerate(rp.reqs):
        ticks = {}
        for task in rp.tasks:
            for row in task.rows:
                if row.rid == rid:
                    ticks[row.node] = (task.tick, task.finish, task.index)
        for v in range(1, len(ticks)):
            assert ticks[v][2] > ticks[v - 1][2]
