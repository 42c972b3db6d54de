"""P9 on CPU: the C++ engine's scheduler (libbm.so, BM_CLOCK_DRY: no device work) produces
exactly the task log, slot indices and completion order/ticks of the independent Python replay
of Algorithm 1 (oracle/scheduler.py) for the same arrival trace."""
import numpy as np
import pytest
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

from oracle.scheduler import CHAIN, SEQ2SEQ, TREE, Replay
from paper_conf_eurosys_gaoywl18_b200 import bm
from workloads import gen

H = 64
V = 16


def _engine(cts, clock=bm.CLOCK_DRY, **kw):
    """cts: list of (kind, bmax, priority). Weights are zeros (DRY: never used)."""
    e = bm.Engine(clock=clock, hidden=H, pool_layers=2, **kw)
    ids = []
    for kind, bmax, prio in cts:
        if kind == bm.CELL_TREE_LEAF:
            W, b, E = [np.zeros((3 * H, H), np.float32)], [np.zeros(3 * H, np.float32)], np.zeros((V, H), np.float32)
            ids.append(e.load_cell(kind, 1, V, bmax, prio, W, b, E))
        elif kind == bm.CELL_TREE_INTERNAL:
            ids.append(e.load_cell(kind, 1, V, bmax, prio, [np.zeros((5 * H, 2 * H), np.float32)],
                                   [np.zeros(5 * H, np.float32)]))
        else:
            W = [np.zeros((4 * H, 2 * H), np.float32)] * 2
            b = [np.zeros(4 * H, np.float32)] * 2
            kw2 = {}
            if kind == bm.CELL_LSTM_PROJ:
                kw2 = dict(W_out=np.zeros((128, H), np.float32), b_out=np.zeros(128, np.float32))
            ids.append(e.load_cell(kind, 2, 128 if kind == bm.CELL_LSTM_PROJ else V, bmax, prio, W, b,
                                   np.zeros((128 if kind == bm.CELL_LSTM_PROJ else V, H), np.float32), **kw2))
    return e, ids


def _submit_all(e, reqs):
    for q in reqs:
        if q["kind"] == CHAIN:
            e.submit(bm.REQ_CHAIN, q["cells"][0], 0, [3] * q["length"], q["arrival"])
        elif q["kind"] == SEQ2SEQ:
            eos = q.get("eos_step")
            e.submit(bm.REQ_SEQ2SEQ, q["cells"][0], q["cells"][1], [3] * q["length"], q["arrival"],
                     decode_len=q["decode_len"], eos_id=5 if "eos_step" in q else None,
                     dry_eos_step=-1 if eos is None else eos)
        else:
            n = len(q["left"])
            e.submit(bm.REQ_TREE, q["cells"][0], q["cells"][1], [3] * n, q["arrival"],
                     left=q["left"], right=q["right"])


def _compare(e, rp):
    log = e.read_log()
    assert len(log) == len(rp.tasks)
    for a, t in zip(log, rp.tasks):
        assert a["cell"] == t.ct
        assert a["tick"] == t.tick
        assert a["worker"] == t.worker
        assert a["rows"] == [(r.rid, r.node, r.slot) for r in t.rows]
    comp = e.poll()
    assert [(c.req_id, c.t_done) for c in comp] == [(rid, float(tk)) for rid, tk in rp.completions]
    for c in comp:
        r = rp.reqs[c.req_id]
        assert c.t_first == r.first_tick


def _chain_case(trace, bmax, minf, max_tasks=5, k=0, slots=1 << 12):
    e, ids = _engine([(bm.CELL_LSTM, bmax, 0)], max_slots=slots, max_requests=1 << 12,
                     min_followon_batch=minf, max_tasks_to_submit=max_tasks,
                     schedule_when_outstanding_leq=k)
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    _submit_all(e, reqs)
    e.run()
    rp = Replay([(bmax, 0)], max_slots=slots, max_tasks_to_submit=max_tasks, min_followon=minf,
                schedule_when_outstanding_leq=k).run(reqs)
    _compare(e, rp)


@pytest.mark.parametrize("minf", [1, 4])
def test_figure5_replay(minf):
    _chain_case(gen.figure5_trace(), 4, minf)


@pytest.mark.parametrize("minf", [1, 4])
def test_config0_replay(minf):
    _chain_case(gen.config0_trace(), 4, minf)


def test_wmt_poisson_replay():
    trace = gen.chain_trace(400, 64, 7, rate=3.0)
    _chain_case(trace, 32, 1, k=2, slots=64)


def test_complete_tree_replay():
    left, right = gen.complete_tree(16)
    reqs = [{"kind": TREE, "cells": [0, 1], "arrival": 0, "left": left, "right": right}]
    e, _ = _engine([(bm.CELL_TREE_LEAF, 64, 0), (bm.CELL_TREE_INTERNAL, 64, 1)], max_slots=256,
                   max_requests=16)
    _submit_all(e, reqs)
    e.run()
    _compare(e, Replay([(64, 0), (64, 1)], max_slots=256).run(reqs))


def _random_reqs(seed, n, kinds, eos=False):
    rng = np.random.default_rng(seed)
    out = []
    t = 0.0
    for _ in range(n):
        t += float(rng.integers(0, 3))
        kind = kinds[int(rng.integers(0, len(kinds)))]
        if kind == CHAIN:
            out.append({"kind": CHAIN, "cells": [0], "arrival": t, "length": int(rng.integers(1, 9))})
        elif kind == SEQ2SEQ:
            q = {"kind": SEQ2SEQ, "cells": [1, 2], "arrival": t,
                 "length": int(rng.integers(1, 6)), "decode_len": int(rng.integers(1, 9))}
            if eos:  # <eos> at a random step, or never (N1)
                st_ = int(rng.integers(0, q["decode_len"] + 2))
                q["eos_step"] = st_ if st_ < q["decode_len"] else None
            out.append(q)
        else:
            left, right = gen._random_bracketing(int(rng.integers(1, 9)), rng)
            out.append({"kind": TREE, "cells": [3, 4], "arrival": t, "left": left, "right": right})
    return out


@settings(max_examples=200, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 100_000), n=st.integers(1, 20),
       bmax=st.lists(st.integers(1, 6), min_size=5, max_size=5),
       prio=st.permutations([0, 1, 2, 3, 4]), max_tasks=st.integers(1, 5),
       min_followon=st.integers(1, 4), k=st.integers(0, 3), slots=st.integers(4, 40),
       kinds=st.sampled_from([[CHAIN], [SEQ2SEQ], [TREE], [CHAIN, SEQ2SEQ, TREE]]))
def test_random_traces_bit_exact(seed, n, bmax, prio, max_tasks, min_followon, k, slots, kinds):
    reqs = _random_reqs(seed, n, kinds)
    need = max((len(q["left"]) if q["kind"] == TREE else 1) for q in reqs)
    slots = max(slots, need)
    kinds_c = [bm.CELL_LSTM, bm.CELL_LSTM, bm.CELL_LSTM_PROJ, bm.CELL_TREE_LEAF, bm.CELL_TREE_INTERNAL]
    e, _ = _engine(list(zip(kinds_c, bmax, prio)), max_slots=slots, max_requests=64,
                   max_tasks_to_submit=max_tasks, min_followon_batch=min_followon,
                   schedule_when_outstanding_leq=k)
    _submit_all(e, reqs)
    e.run()
    rp = Replay(list(zip(bmax, prio)), max_slots=slots, max_tasks_to_submit=max_tasks,
                min_followon=min_followon, schedule_when_outstanding_leq=k).run(reqs)
    _compare(e, rp)


def test_schedule_step_api_matches_run():
    """Driving the engine with bm_schedule_step (the paper's per-idle Schedule call) gives the
    same log as bm_run."""
    trace = gen.config0_trace()
    e, _ = _engine([(bm.CELL_LSTM, 4, 0)], max_slots=16, max_requests=16)
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": q.arrival, "length": q.length} for q in trace]
    _submit_all(e, reqs)
    n = 0
    while e.schedule_step() >= 0:
        n += 1
        assert n < 1000
    rp = Replay([(4, 0)], max_slots=16).run(reqs)
    _compare(e, rp)


@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 100_000), n=st.integers(1, 16),
       bmax=st.lists(st.integers(1, 6), min_size=5, max_size=5),
       prio=st.permutations([0, 1, 2, 3, 4]), max_tasks=st.integers(1, 5),
       k=st.integers(0, 3), slots=st.integers(4, 40),
       kinds=st.sampled_from([[SEQ2SEQ], [CHAIN, SEQ2SEQ, TREE]]))
def test_random_eos_traces_bit_exact(seed, n, bmax, prio, max_tasks, k, slots, kinds):
    """§8f N1: <eos>-terminated decoding. The engine learns each request's <eos> at the retire
    of the task that emitted it (BM_CLOCK_DRY: reported via dry_eos_step) and stops scheduling
    its decoder; the replay follows the same rule independently. Logs and completions equal."""
    reqs = _random_reqs(seed, n, kinds, eos=True)
    need = max((len(q["left"]) if q["kind"] == TREE else 1) for q in reqs)
    slots = max(slots, need)
    kinds_c = [bm.CELL_LSTM, bm.CELL_LSTM, bm.CELL_LSTM_PROJ, bm.CELL_TREE_LEAF, bm.CELL_TREE_INTERNAL]
    e, _ = _engine(list(zip(kinds_c, bmax, prio)), max_slots=slots, max_requests=64,
                   max_tasks_to_submit=max_tasks, schedule_when_outstanding_leq=k)
    _submit_all(e, reqs)
    e.run()
    rp = Replay(list(zip(bmax, prio)), max_slots=slots, max_tasks_to_submit=max_tasks,
                schedule_when_outstanding_leq=k).run(reqs)
    _compare(e, rp)


def test_eos_request_rejected_when_invalid():
    e, ids = _engine([(bm.CELL_LSTM, 4, 0), (bm.CELL_LSTM_PROJ, 4, 1)], max_slots=16, max_requests=16)
    with pytest.raises(RuntimeError):
        e.submit(bm.REQ_SEQ2SEQ, ids[0], ids[1], [3, 4], 0, decode_len=4, eos_id=128)  # >= vocab
    with pytest.raises(RuntimeError):
        e.submit(bm.REQ_SEQ2SEQ, ids[0], ids[1], [3, 4], 0, decode_len=4, eos_id=-2)


@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 100_000), n=st.integers(1, 20),
       bmax=st.lists(st.integers(1, 6), min_size=5, max_size=5),
       prio=st.permutations([0, 1, 2, 3, 4]), max_tasks=st.integers(1, 5),
       k=st.integers(0, 3), slots=st.integers(4, 40), workers=st.integers(2, 4),
       kinds=st.sampled_from([[CHAIN], [SEQ2SEQ], [TREE], [CHAIN, SEQ2SEQ, TREE]]), eos=st.booleans())
def test_multi_worker_traces_bit_exact(seed, n, bmax, prio, max_tasks, k, slots, workers, kinds, eos):
    """§8f N2: one manager, W workers (L317): Schedule(worker) for each idle worker, subgraphs
    pinned to the worker running them (Alg. 1 lines 21, 27; unpinned at in-flight 0, L381).
    The engine (W streams) and the replay agree task for task, worker for worker."""
    reqs = _random_reqs(seed, n, kinds, eos=eos)
    need = max((len(q["left"]) if q["kind"] == TREE else 1) for q in reqs)
    slots = max(slots, need)
    kinds_c = [bm.CELL_LSTM, bm.CELL_LSTM, bm.CELL_LSTM_PROJ, bm.CELL_TREE_LEAF, bm.CELL_TREE_INTERNAL]
    e, _ = _engine(list(zip(kinds_c, bmax, prio)), max_slots=slots, max_requests=64,
                   max_tasks_to_submit=max_tasks, schedule_when_outstanding_leq=k, workers=workers)
    _submit_all(e, reqs)
    e.run()
    rp = Replay(list(zip(bmax, prio)), max_slots=slots, max_tasks_to_submit=max_tasks,
                schedule_when_outstanding_leq=k, workers=workers).run(reqs)
    _compare(e, rp)


def test_submit_rejects_arrival_before_pending():
    """Reading S21 / L323: each request is admitted at its own arrival. The boundary takes an
    arrival stream: a request may not arrive before one still pending (BM_E_INVAL), so the
    engine's FIFO admission is exactly "every due arrival, in trace order"."""
    e, (cid,) = _engine([(bm.CELL_LSTM, 4, 0)], max_slots=64, max_requests=64)
    e.submit(bm.REQ_CHAIN, cid, 0, [3, 3], 2.0)
    with pytest.raises(bm.BMError):
        e.submit(bm.REQ_CHAIN, cid, 0, [3], 1.0)
    e.submit(bm.REQ_CHAIN, cid, 0, [3], 2.0)   # equal arrival: fine
    e.run()
    assert len(e.poll()) == 2
    e.submit(bm.REQ_CHAIN, cid, 0, [3], 0.0)   # nothing pending any more: any arrival
    e.run()
    assert len(e.poll()) == 1


def test_replay_admits_due_arrivals_in_trace_order():
    """The replay admits every request whose arrival has passed, in trace order, whatever the
    order of later entries (L323): a late-listed early arrival is not held back behind an
    earlier-listed late one."""
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": 3.0, "length": 1},
            {"kind": CHAIN, "cells": [0], "arrival": 0.0, "length": 1}]
    rp = Replay([(4, 0)], max_slots=8).run(reqs)
    assert rp.tasks[0].tick == 0.0 and len(rp.tasks[0].rows) == 1
    assert sorted(t for _, t in rp.completions) == [1.0, 4.0]


@settings(max_examples=150, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(seed=st.integers(0, 100_000), n=st.integers(1, 20),
       bmax=st.lists(st.integers(1, 6), min_size=5, max_size=5),
       prio=st.permutations([0, 1, 2, 3, 4]), max_tasks=st.integers(1, 5),
       k=st.integers(0, 3), slots=st.integers(4, 40), workers=st.integers(2, 4), devices=st.integers(2, 4),
       kinds=st.sampled_from([[CHAIN], [SEQ2SEQ], [TREE], [CHAIN, SEQ2SEQ, TREE]]), eos=st.booleans())
def test_multi_device_traces_bit_exact(seed, n, bmax, prio, max_tasks, k, slots, workers, devices, kinds, eos):
    """§8f N2 across GPUs (L317, L337): W workers spread over D device contexts (worker w on
    context w % D). Scheduling is Algorithm 1 as with one device -- the task log (worker by
    worker), slots and completions equal the replay -- and the state rows moved between
    contexts (an unpinned subgraph scheduled on another device, L337/L381; tree children
    computed elsewhere) are exactly the replay's count."""
    devices = min(devices, workers)
    reqs = _random_reqs(seed, n, kinds, eos=eos)
    need = max((len(q["left"]) if q["kind"] == TREE else 1) for q in reqs)
    slots = max(slots, need)
    kinds_c = [bm.CELL_LSTM, bm.CELL_LSTM, bm.CELL_LSTM_PROJ, bm.CELL_TREE_LEAF, bm.CELL_TREE_INTERNAL]
    e, _ = _engine(list(zip(kinds_c, bmax, prio)), max_slots=slots, max_requests=64,
                   max_tasks_to_submit=max_tasks, schedule_when_outstanding_leq=k, workers=workers,
                   devices=devices)
    _submit_all(e, reqs)
    e.run()
    rp = Replay(list(zip(bmax, prio)), max_slots=slots, max_tasks_to_submit=max_tasks,
                schedule_when_outstanding_leq=k, workers=workers, devices=devices).run(reqs)
    _compare(e, rp)
    assert e.stats()["migrations"] == rp.migrations


def test_multi_device_migrations_happen():
    """A hand-checkable case: three 3-step chain requests arriving at ticks 0, 1, 2, bmax 1,
    MaxTasksToSubmit 1, two workers on two device contexts. Worker 1 runs request 1's first two
    steps; at tick 3 request 1 is unpinned and worker 0 (first in id order) takes its last step
    -> one move; request 2 starts on worker 1 and continues on worker 0 -> a second move."""
    reqs = [{"kind": CHAIN, "cells": [0], "arrival": float(i), "length": 3} for i in range(3)]
    e, _ = _engine([(bm.CELL_LSTM, 1, 0)], max_slots=8, max_requests=8, workers=2, devices=2,
                   max_tasks_to_submit=1)
    _submit_all(e, reqs)
    e.run()
    rp = Replay([(1, 0)], max_slots=8, workers=2, devices=2, max_tasks_to_submit=1).run(reqs)
    _compare(e, rp)
    assert [(t.worker, [(r.rid, r.node) for r in t.rows]) for t in rp.tasks][5:7] == [(0, [(1, 2)]), (1, [(2, 0)])]
    assert e.stats()["migrations"] == rp.migrations == 2
