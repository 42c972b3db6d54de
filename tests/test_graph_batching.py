"""N4, the padding + bucketing graph-batching baseline (§7.1) as a policy of
the same engine: its replay oracle pinned to the paper's statements, and the C++ engine's task
log / completions bit-exact with the replay (CPU, BM_CLOCK_DRY)."""
import numpy as np
import pytest
from hypothesis import given, settings
from hypothesis import strategies as st

from oracle.scheduler import GraphBatchingReplay
from paper_conf_eurosys_gaoywl18_b200 import bm

H, V = 64, 16


def _replay(lengths, arrivals, bmax=4, w=10, k=0, slots=1 << 20):
    rp = GraphBatchingReplay(bmax, max_slots=slots, bucket_width=w, schedule_when_outstanding_leq=k)
    return rp.run([dict(arrival=a, length=L) for a, L in zip(arrivals, lengths)])


def test_pin_padding_to_bucket_bound():
    """L631: "a request of length 21 will be padded to length 30" (bucket width 10)."""
    rp = _replay([21], [0])
    assert len(rp.tasks) == 30
    assert all(len(t.rows) == 1 for t in rp.tasks)
    assert rp.completions == [(0, 30.0)]


def test_pin_33_buckets():
    """L427: max length 330, width 10 -> 33 buckets; bucket i holds (i*10, (i+1)*10]."""
    rp = GraphBatchingReplay(4, bucket_width=10)
    assert {rp.bucket(L) for L in range(1, 331)} == set(range(33))
    assert rp.bucket(10) == 0 and rp.bucket(11) == 1 and rp.bucket(330) == 32


def test_pin_hand_computed_round_robin():
    """Five requests at t=0, bmax 4: bucket 0 (3, 5, 8) runs 10 steps, then bucket 1 (12) 20,
    then bucket 2 (21) 30; every request of a batch returns at the batch's end (L631 'jumps')."""
    rp = _replay([3, 21, 5, 12, 8], [0] * 5)
    assert rp.completions == [(0, 10.0), (2, 10.0), (4, 10.0), (3, 30.0), (1, 60.0)]
    assert [len(t.rows) for t in rp.tasks] == [3] * 10 + [1] * 20 + [1] * 30


@settings(max_examples=60, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 45), st.integers(0, 40)), min_size=1, max_size=25),
       st.integers(1, 6), st.integers(1, 12), st.integers(0, 2))
def test_pin_invariants(reqs, bmax, w, k):
    """Every request runs in exactly one batch padded to its bucket bound, batches <= bmax and
    single-bucket, all of a batch complete together, round robin never serves a bucket twice
    while another non-empty bucket waits longer in cyclic order."""
    reqs = sorted(reqs, key=lambda x: x[1])
    lengths = [L for L, _ in reqs]
    arrivals = [float(a) for _, a in reqs]
    rp = _replay(lengths, arrivals, bmax=bmax, w=w, k=k)
    seen = {}
    batches = []
    i = 0
    while i < len(rp.tasks):
        rows = [r.rid for r in rp.tasks[i].rows]
        bkt = {(lengths[r] - 1) // w for r in rows}
        assert len(bkt) == 1 and len(rows) <= bmax
        steps = (bkt.pop() + 1) * w
        for s in range(steps):
            assert [r.rid for r in rp.tasks[i + s].rows] == rows
            assert all(r.node == s for r in rp.tasks[i + s].rows)
        batches.append(rows)
        for r in rows:
            assert r not in seen
            seen[r] = len(batches) - 1
        i += steps
    assert sorted(seen) == list(range(len(lengths)))
    done = dict(rp.completions)
    for rows in batches:
        assert len({done[r] for r in rows}) == 1


def _engine(bmax=4, w=10, k=0, slots=4096):
    e = bm.Engine(clock=bm.CLOCK_DRY, hidden=H, pool_layers=1, policy=bm.POLICY_GRAPH, bucket_width=w,
                  schedule_when_outstanding_leq=k, max_slots=slots)
    cid = e.load_cell(bm.CELL_LSTM, 1, V, bmax, 0, [np.zeros((4 * H, 2 * H), np.float32)],
                      [np.zeros(4 * H, np.float32)], np.zeros((V, H), np.float32))
    return e, cid


def _compare(e, rp):
    log = e.read_log()
    assert len(log) == len(rp.tasks)
    for a, t in zip(log, rp.tasks):
        assert a["tick"] == t.tick
        assert a["rows"] == [(r.rid, r.node, r.slot) for r in t.rows]
    comp = e.poll()
    assert [(c.req_id, c.t_done) for c in comp] == [(rid, float(tk)) for rid, tk in rp.completions]


@settings(max_examples=60, deadline=None)
@given(st.lists(st.tuples(st.integers(1, 45), st.integers(0, 60)), min_size=1, max_size=30),
       st.integers(1, 6), st.integers(1, 12), st.integers(0, 2), st.integers(2, 64))
def test_engine_matches_replay(reqs, bmax, w, k, slots):
    reqs = sorted(reqs, key=lambda x: x[1])
    e, cid = _engine(bmax, w, k, slots)
    for L, a in reqs:
        e.submit(bm.REQ_CHAIN, cid, 0, [3] * L, float(a))
    assert e.run() == len(reqs)
    rp = _replay([L for L, _ in reqs], [float(a) for _, a in reqs], bmax=bmax, w=w, k=k, slots=slots)
    _compare(e, rp)
    e.close()


def test_graph_policy_rejects_non_chain():
    e, cid = _engine()
    with pytest.raises(bm.BMError):
        e.submit(bm.REQ_TREE, cid, cid, [3, 3, 3], 0.0, left=np.array([-1, -1, 0]), right=np.array([-1, -1, 1]))
    e.close()
