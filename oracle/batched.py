"""fp64 *batched* executor: runs an explicit schedule of batched tasks, each task executing
its rows as one stacked matrix contraction, exactly as cellular batching does (§3.1:
cells of the same type with no data dependency between them are batched together).

TEST INFRASTRUCTURE ONLY. Used by tests/test_oracle_batching.py (pin P4) to check by brute
force that every dependency-respecting batching schedule reaches the unbatched result of
oracle.cells (the method is exact: batching only concatenates independent rows).
"""
from __future__ import annotations

from typing import Dict, List, Sequence, Tuple

import numpy as np

from .cells import f64, sigmoid


def _lstm_rows(W, b, X, Hp, Cp):
    H = Hp.shape[1]
    Z = np.concatenate([X, Hp], axis=1) @ f64(W).T + f64(b)
    i, f = sigmoid(Z[:, :H]), sigmoid(Z[:, H:2 * H])
    g, o = np.tanh(Z[:, 2 * H:3 * H]), sigmoid(Z[:, 3 * H:])
    C = f * Cp + i * g
    return o * np.tanh(C), C


def run_chain_schedule(w, token_lists: Sequence[Sequence[int]],
                       schedule: Sequence[Sequence[Tuple[int, int]]]):
    """schedule: list of tasks, each a list of (request, step) rows. Single-layer or stacked
    LSTM: each row runs one full timestep of the stack. Returns {request: (h list, c list)}."""
    Hd, L = w.hidden, w.layers
    h = {r: [np.zeros(Hd) for _ in range(L)] for r in range(len(token_lists))}
    c = {r: [np.zeros(Hd) for _ in range(L)] for r in range(len(token_lists))}
    done = {r: 0 for r in range(len(token_lists))}
    for task in schedule:
        rows = list(task)
        for r, k in rows:
            assert done[r] == k, "schedule violates chain order"
        X = np.stack([f64(w.E[int(token_lists[r][k])]) for r, k in rows])
        for l in range(L):
            Hp = np.stack([h[r][l] for r, _ in rows])
            Cp = np.stack([c[r][l] for r, _ in rows])
            Hn, Cn = _lstm_rows(w.W[l], w.b[l], X, Hp, Cp)
            for j, (r, _) in enumerate(rows):
                h[r][l], c[r][l] = Hn[j], Cn[j]
            X = Hn
        for r, _ in rows:
            done[r] += 1
    return {r: (h[r], c[r]) for r in h}


def run_tree_schedule(w, trees: Sequence[Tuple[Sequence[int], Sequence[int], Sequence[int]]],
                      schedule: Sequence[Sequence[Tuple[int, int]]]):
    """trees: list of (tokens, left, right) in post-order. schedule: tasks of (tree, node)
    rows; a task holds only leaves or only internal nodes (two cell types, L99, L383).
    Returns {tree: (root_h, root_c)}."""
    Hd = w.hidden
    st: Dict[Tuple[int, int], Tuple[np.ndarray, np.ndarray]] = {}
    for task in schedule:
        rows = list(task)
        leaf = [trees[t][1][v] < 0 for t, v in rows]
        assert all(leaf) or not any(leaf), "mixed cell types in one task"
        if all(leaf):
            X = np.stack([f64(w.E[int(trees[t][0][v])]) for t, v in rows])
            Z = X @ f64(w.W_leaf).T + f64(w.b_leaf)
            i, o, u = sigmoid(Z[:, :Hd]), sigmoid(Z[:, Hd:2 * Hd]), np.tanh(Z[:, 2 * Hd:])
            C = i * u
            Hn = o * np.tanh(C)
        else:
            for t, v in rows:
                assert (t, trees[t][1][v]) in st and (t, trees[t][2][v]) in st, "dependency"
            HL = np.stack([st[(t, trees[t][1][v])][0] for t, v in rows])
            CL = np.stack([st[(t, trees[t][1][v])][1] for t, v in rows])
            HR = np.stack([st[(t, trees[t][2][v])][0] for t, v in rows])
            CR = np.stack([st[(t, trees[t][2][v])][1] for t, v in rows])
            Z = np.concatenate([HL, HR], axis=1) @ f64(w.U).T + f64(w.b_int)
            i, fL, fR = sigmoid(Z[:, :Hd]), sigmoid(Z[:, Hd:2 * Hd]), sigmoid(Z[:, 2 * Hd:3 * Hd])
            o, u = sigmoid(Z[:, 3 * Hd:4 * Hd]), np.tanh(Z[:, 4 * Hd:])
            C = i * u + fL * CL + fR * CR
            Hn = o * np.tanh(C)
        for j, (t, v) in enumerate(rows):
            st[(t, v)] = (Hn[j], C[j])
    return {t: st[(t, len(trees[t][1]) - 1)] for t in range(len(trees))}


def run_seq2seq_forced_lockstep(enc, dec, srcs: Sequence[Sequence[int]],
                                forced: Sequence[Sequence[int]], chunk: int = 1024):
    """Seq2Seq in forced-token mode (decoding per L713-L715) for many requests at
    once, in lockstep: encoder step k batches every request with > k source tokens; decoder
    step s batches every request with > s decode steps and feeds <go> at s = 0, else the given
    token forced[r][s-1]. Exactly the rows-concatenation of cells.seq2seq(..., forced_tokens)
    (pinned against it in tests/test_oracle_batching.py).

    Returns (h, c, sel, best): h, c = per request lists of per-layer final states; sel[r][s] =
    logit of the forced (emitted) token forced[r][s] at step s, best[r][s] = max logit there
    (for the argmax-validity check; the full logits are not kept)."""
    from .cells import GO
    n, Hd, L = len(srcs), enc.hidden, enc.layers
    h = [np.zeros((n, Hd)) for _ in range(L)]
    c = [np.zeros((n, Hd)) for _ in range(L)]

    def stack_step(w, rows, X):
        for l in range(L):
            Hn, Cn = _lstm_rows(w.W[l], w.b[l], X, h[l][rows], c[l][rows])
            h[l][rows], c[l][rows] = Hn, Cn
            X = Hn
        return X

    S = np.array([len(s) for s in srcs])
    for k in range(int(S.max())):
        rows = np.flatnonzero(S > k)
        stack_step(enc, rows, np.stack([f64(enc.E[int(srcs[r][k])]) for r in rows]))
    T = np.array([len(f) for f in forced])
    sel = [np.zeros(t) for t in T]
    best = [np.zeros(t) for t in T]
    Wo, bo = f64(dec.W_out), f64(dec.b_out)
    for s in range(int(T.max())):
        rows = np.flatnonzero(T > s)
        toks = [GO if s == 0 else int(forced[r][s - 1]) for r in rows]
        top = stack_step(dec, rows, np.stack([f64(dec.E[t]) for t in toks]))
        for a in range(0, len(rows), chunk):
            Z = top[a:a + chunk] @ Wo.T + bo
            for j, r in enumerate(rows[a:a + chunk]):
                sel[r][s] = Z[j, int(forced[r][s])]
                best[r][s] = Z[j].max()
    return ([[h[l][r] for l in range(L)] for r in range(n)],
            [[c[l][r] for l in range(L)] for r in range(n)], sel, best)


def lstm_step_rows(W, b, X, Hp, Cp):
    """One LSTM step (reading S1) for a stack of independent rows: X, Hp, Cp [rows, h] -> (H', C').
    The row-stacked form of cells.lstm_cell that run_chain_schedule applies per task."""
    return _lstm_rows(W, b, f64(X), f64(Hp), f64(Cp))
