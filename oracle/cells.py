"""fp64 CPU oracle for the cell maths of cellular batching.

TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
--impl reference legs may import this module. The product path (the C-ABI library and its
Python binding) never imports, calls or links anything under oracle/.

Every function runs ONE request alone, step by step, in float64 (numpy), exactly as the
method defines it: cellular batching is exact, batching only concatenates independent rows
(§3.1), so the unbatched result is the definition the batched GPU path must reach.

The paper prints no cell equations; it cites the LSTM [24] (L105), TreeLSTM [39] (L99) and
gives the LSTM contraction shape b x 2h . 2h x 4h (footnote 2, L205). Readings (DESIGN.md,
SURVEY.md §8c S1-S11):
  S1  LSTM: z = W [x; h] + b, gate row blocks (i, f, g, o); i,f,o = sigmoid, g = tanh;
      c' = f*c + i*g ; h' = o*tanh(c'). No peepholes, no forget-bias offset.
  S2  h0 = c0 = 0.
  S3  x = E[token], E is [V, h].
  S6  Seq2Seq: L-layer encoder and L-layer decoder, one cell = one timestep of the stack.
  S7  decoder layer l starts from encoder layer l's final (h, c).
  S8/S9 greedy feed-previous for exactly T steps (L715); argmax ties -> lowest index.
  N1  optional <eos> stop: the step emitting <eos> is the last, T is then the maximum (L715).
  S10 logits = W_out h_L + b_out.
  S11 TreeLSTM (binary N-ary form): leaf z = W_leaf x + b -> (i, o, u), c = i*u,
      h = o*tanh(c); internal z = U [h_L; h_R] + b -> (i, f_L, f_R, o, u),
      c = i*u + f_L*c_L + f_R*c_R, h = o*tanh(c), with i,f,o = sigmoid, u = tanh.

Pins (tests/test_oracle_pins.py): closed form (P1), torch.nn.LSTMCell / nn.LSTM fp64 (P2),
caterpillar reduction + mirror invariance + leaf == LSTMCell(x,0,0) (P3), brute-force
batching equivalence (P4, tests/test_oracle_batching.py).
"""
from __future__ import annotations

from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

GO = 1  # <go> token id (reading S3)


def sigmoid(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        return 1.0 / (1.0 + np.exp(-z))


def f64(a) -> np.ndarray:
    return np.asarray(a, dtype=np.float64)


# ---------------------------------------------------------------- LSTM (M1; L105, L205)

def lstm_cell(W: np.ndarray, b: np.ndarray, x: np.ndarray, h: np.ndarray, c: np.ndarray
              ) -> Tuple[np.ndarray, np.ndarray]:
    """One LSTM step (reading S1). W [4h, 2h] acts on the column [x; h] (footnote 2, L205)."""
    H = h.shape[0]
    z = f64(W) @ np.concatenate([f64(x), f64(h)]) + f64(b)
    i = sigmoid(z[0:H])
    f = sigmoid(z[H:2 * H])
    g = np.tanh(z[2 * H:3 * H])
    o = sigmoid(z[3 * H:4 * H])
    c_new = f * f64(c) + i * g
    h_new = o * np.tanh(c_new)
    return h_new, c_new


def lstm_stack_step(Ws: Sequence[np.ndarray], bs: Sequence[np.ndarray], x: np.ndarray,
                    hs: List[np.ndarray], cs: List[np.ndarray]):
    """One timestep of an L-layer stack: the input of layer l is h' of layer l-1 (A11)."""
    new_h, new_c = [], []
    inp = f64(x)
    for l in range(len(Ws)):
        hn, cn = lstm_cell(Ws[l], bs[l], inp, hs[l], cs[l])
        new_h.append(hn)
        new_c.append(cn)
        inp = hn
    return new_h, new_c


def chain_lstm(w, tokens: Sequence[int]):
    """Chain LSTM application (M2, Fig. 1 L77-L81): x_t = E[tok_t] for t = 1..L.
    Returns final per-layer (h, c) lists (reading S5: no output projection)."""
    H = w.hidden
    hs = [np.zeros(H) for _ in range(w.layers)]
    cs = [np.zeros(H) for _ in range(w.layers)]
    for tok in tokens:
        hs, cs = lstm_stack_step(w.W, w.b, f64(w.E[int(tok)]), hs, cs)
    return hs, cs


# ---------------------------------------------------------------- Seq2Seq (M3/M4; L685-L721)

def argmax_lowest(v: np.ndarray) -> int:
    """argmax with ties resolved to the lowest index (reading S9)."""
    return int(np.flatnonzero(v == v.max())[0])


def seq2seq(enc, dec, src_tokens: Sequence[int], decode_len: int,
            forced_tokens: Optional[Sequence[int]] = None, eos_id: Optional[int] = None) -> Dict[str, object]:
    """Encoder over the source, then greedy feed-previous decoding (L713-L715).

    eos_id None: exactly decode_len steps (the paper's evaluation protocol, L715).
    eos_id set: "Decoding terminates when either the <eos> symbol is generated or when the
    maximum decoding length is reached" (L715, deployed systems) -- decode_len is then the
    maximum length; the step that emits <eos> is the last one (its state is the result).

    If forced_tokens is given (the GPU's emitted tokens, SURVEY §8c "forced-token mode") the
    decoder feeds those instead of its own argmax -- and termination follows them too -- so
    that a legitimate bf16 argmax flip does not desynchronise the comparison; the oracle's
    own argmax is still returned for the validity check."""
    hs, cs = chain_lstm(enc, src_tokens)
    logits_all, own_tokens, fed = [], [], []
    prev = GO
    for s in range(decode_len):
        hs, cs = lstm_stack_step(dec.W, dec.b, f64(dec.E[int(prev)]), hs, cs)
        logits = f64(dec.W_out) @ hs[-1] + f64(dec.b_out)
        y = argmax_lowest(logits)
        logits_all.append(logits)
        own_tokens.append(y)
        prev = int(forced_tokens[s]) if forced_tokens is not None else y
        fed.append(prev)
        if eos_id is not None and prev == eos_id:
            break
    return {"h": hs, "c": cs, "logits": np.array(logits_all), "tokens": own_tokens,
            "fed_tokens": fed}


# ---------------------------------------------------------------- TreeLSTM (M5/M6; L99, L383)

def tree_leaf(W_leaf, b_leaf, x):
    H = W_leaf.shape[1]
    z = f64(W_leaf) @ f64(x) + f64(b_leaf)
    i = sigmoid(z[0:H])
    o = sigmoid(z[H:2 * H])
    u = np.tanh(z[2 * H:3 * H])
    c = i * u
    h = o * np.tanh(c)
    return h, c


def tree_internal(U, b_int, hL, cL, hR, cR):
    H = hL.shape[0]
    z = f64(U) @ np.concatenate([f64(hL), f64(hR)]) + f64(b_int)
    i = sigmoid(z[0:H])
    fL = sigmoid(z[H:2 * H])
    fR = sigmoid(z[2 * H:3 * H])
    o = sigmoid(z[3 * H:4 * H])
    u = np.tanh(z[4 * H:5 * H])
    c = i * u + fL * f64(cL) + fR * f64(cR)
    h = o * np.tanh(c)
    return h, c


def tree_lstm(w, tokens: Sequence[int], left: Sequence[int], right: Sequence[int]):
    """Evaluate a binary tree given in post-order (children before parents, root last).
    Returns (root_h, root_c, per-node list of (h, c))."""
    n = len(left)
    states: List[Tuple[np.ndarray, np.ndarray]] = [None] * n  # type: ignore
    for v in range(n):
        if left[v] < 0:
            states[v] = tree_leaf(w.W_leaf, w.b_leaf, f64(w.E[int(tokens[v])]))
        else:
            hL, cL = states[left[v]]
            hR, cR = states[right[v]]
            states[v] = tree_internal(w.U, w.b_int, hL, cL, hR, cR)
    return states[-1][0], states[-1][1], states
