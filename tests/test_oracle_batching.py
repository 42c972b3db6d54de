"""Pin P4: brute-force batching equivalence.

Cellular batching is exact (§3.1: cells with no data dependency between them
are batched; batching concatenates independent rows). For tiny traces we enumerate EVERY
dependency-respecting sequence of batched tasks (any cell-type-homogeneous set of ready
nodes of size <= bmax), run it through the fp64 batched executor and require the unbatched
oracle result to 1e-12 for every request."""
import itertools

import numpy as np
import pytest

from oracle import batched, cells
from workloads import gen


def _chain_schedules(lengths, bmax, limit=20000):
    """All task sequences for chain requests: a task = subset (<= bmax) of requests that
    still have steps left; each row runs that request's next step."""
    out = []

    def rec(done, seq):
        if len(out) >= limit:
            return
        live = [r for r in range(len(lengths)) if done[r] < lengths[r]]
        if not live:
            out.append(list(seq))
            return
        for k in range(1, min(bmax, len(live)) + 1):
            for sub in itertools.combinations(live, k):
                task = [(r, done[r]) for r in sub]
                nd = list(done)
                for r in sub:
                    nd[r] += 1
                seq.append(task)
                rec(nd, seq)
                seq.pop()

    rec([0] * len(lengths), [])
    return out


@pytest.mark.parametrize("lengths,bmax", [([1, 2], 2), ([2, 3], 1), ([3, 1, 2], 2),
                                          ([2, 2, 3], 3), ([3, 3, 3], 2)])
@pytest.mark.parametrize("layers", [1, 2])
def test_p4_chain_every_schedule_equals_unbatched(lengths, bmax, layers):
    w = gen.lstm_stack_weights(6, layers, 20, seed=len(lengths) * 7 + bmax, bf16=False)
    rng = np.random.default_rng(1)
    toks = [rng.integers(3, 20, size=L) for L in lengths]
    ref = [cells.chain_lstm(w, t) for t in toks]
    scheds = _chain_schedules(lengths, bmax)
    assert len(scheds) > 0
    for s in scheds:
        res = batched.run_chain_schedule(w, toks, s)
        for r in range(len(lengths)):
            for l in range(layers):
                assert np.max(np.abs(res[r][0][l] - ref[r][0][l])) <= 1e-12
                assert np.max(np.abs(res[r][1][l] - ref[r][1][l])) <= 1e-12


def _tree_schedules(trees, bmax, limit=5000):
    """All dependency-respecting task sequences over several trees; a task is a set of
    ready nodes of ONE cell type (leaf or internal), size <= bmax."""
    out = []
    nodes = [(t, v) for t in range(len(trees)) for v in range(len(trees[t][1]))]

    def ready(done):
        rl, ri = [], []
        for t, v in nodes:
            if (t, v) in done:
                continue
            L, R = trees[t][1][v], trees[t][2][v]
            if L < 0:
                rl.append((t, v))
            elif (t, L) in done and (t, R) in done:
                ri.append((t, v))
        return rl, ri

    def rec(done, seq):
        if len(out) >= limit:
            return
        if len(done) == len(nodes):
            out.append(list(seq))
            return
        for group in ready(done):
            for k in range(1, min(bmax, len(group)) + 1):
                for sub in itertools.combinations(group, k):
                    seq.append(list(sub))
                    rec(done | set(sub), seq)
                    seq.pop()

    rec(frozenset(), [])
    return out


@pytest.mark.parametrize("leaves,bmax", [([2], 2), ([3], 2), ([2, 2], 2), ([3, 2], 3), ([4], 3)])
def test_p4_tree_every_schedule_equals_unbatched(leaves, bmax):
    w = gen.tree_weights(6, 20, seed=sum(leaves) + bmax, bf16=False)
    rng = np.random.default_rng(sum(leaves))
    trees = []
    for n in leaves:
        left, right = gen._random_bracketing(n, rng)
        toks = rng.integers(3, 20, size=len(left))
        trees.append((toks, left, right))
    ref = [cells.tree_lstm(w, *tr)[:2] for tr in trees]
    scheds = _tree_schedules(trees, bmax)
    assert len(scheds) > 0
    for s in scheds:
        res = batched.run_tree_schedule(w, trees, s)
        for t in range(len(trees)):
            assert np.max(np.abs(res[t][0] - ref[t][0])) <= 1e-12
            assert np.max(np.abs(res[t][1] - ref[t][1])) <= 1e-12


def test_p4_batched_executor_rejects_dependency_violation():
    """The executor itself refuses schedules that break the cell graph's order, so the
    equivalence above is over valid schedules only."""
    w = gen.lstm_stack_weights(4, 1, 10, seed=0, bf16=False)
    with pytest.raises(AssertionError):
        batched.run_chain_schedule(w, [[3, 4]], [[(0, 1)]])


def test_seq2seq_forced_lockstep_equals_unbatched():
    """oracle.batched.run_seq2seq_forced_lockstep (the full-size Seq2Seq parity check's
    executor) = cells.seq2seq(..., forced_tokens) row by row: final per-layer (h, c) to 1e-12,
    the forced token's logit and the step maximum equal to the unbatched logits. Ragged source
    and decode lengths, forced tokens that differ from the oracle's own argmax."""
    h, L, V = 16, 3, 40
    enc = gen.lstm_stack_weights(h, L, V, 31, bf16=False)
    dec = gen.lstm_stack_weights(h, L, V, 32, projection=True, bf16=False)
    rng = np.random.default_rng(5)
    srcs = [list(rng.integers(3, V, size=n)) for n in (1, 4, 2, 6, 3)]
    forced = [list(rng.integers(0, V, size=t)) for t in (3, 1, 5, 2, 4)]
    H_, C_, sel, best = batched.run_seq2seq_forced_lockstep(enc, dec, srcs, forced, chunk=2)
    for r in range(len(srcs)):
        o = cells.seq2seq(enc, dec, srcs[r], len(forced[r]), forced_tokens=forced[r])
        for l in range(L):
            np.testing.assert_allclose(H_[r][l], o["h"][l], rtol=0, atol=1e-12)
            np.testing.assert_allclose(C_[r][l], o["c"][l], rtol=0, atol=1e-12)
        for s, y in enumerate(forced[r]):
            assert abs(sel[r][s] - o["logits"][s][y]) <= 1e-12
            assert abs(best[r][s] - o["logits"][s].max()) <= 1e-12
