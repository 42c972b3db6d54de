"""Seeded synthetic workload generators shared by the oracle, the tests and bench.py.

This module holds NO arithmetic of the method (no cell maths, no scheduling). It only
draws random numbers and shapes them like the paper's workloads, so that both the
CUDA path and the fp64 oracle can be fed the same inputs.

Paper passages the shapes follow (PAPER.md line numbers):
  * hidden size 1024 for every cell ........................... L419 (§7.1)
  * WMT-15 lengths: mean 24, max 330, ~99% < 100 .............. L421, L635 (§7.1, Fig. 10)
  * Poisson inter-arrival times ............................... L423 (§7.1)
  * TreeBank: binary parse trees .............................. L421, L817 (§7.5)
  * identical complete binary tree with 16 leaves ............. L857 (Fig. 15)
  * Figure 5 eight-request example ............................ L223-L271 (§3.2)
Readings where the paper is silent are SURVEY.md §8(c) S3, S4, S25, S26 and are listed in
DESIGN.md.
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional, Sequence

import numpy as np

# Token ids (reading S3): 0 = pad, 1 = <go>, 2 = <eos>, payload tokens in [3, V).
PAD, GO, EOS = 0, 1, 2
FIRST_PAYLOAD = 3

# Request kinds (mirrors include/bm.h BM_REQ_*; plain integers, no behaviour).
CHAIN, SEQ2SEQ, TREE = 0, 1, 2


def bf16_round(x: np.ndarray) -> np.ndarray:
    """Round fp32 values to the nearest bf16-representable fp32 (round-to-nearest-even), with
    magnitudes below 2^-14 (fp16's smallest normal) flushed to zero.

    Used only to make generated values exactly representable on the tensor-core path, which
    holds bf16-valued weights and its activations in fp16 storage (precision):
    a bf16 value of magnitude >= 2^-14 is exact in fp16, so the device and the fp64 oracle see
    identical values (reading S25)."""
    a = np.ascontiguousarray(x, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    u = (u + 0x7FFF + lsb) & 0xFFFF0000
    r = u.astype(np.uint32).view(np.float32).reshape(a.shape)
    return np.where(np.abs(r) < 2.0 ** -14, np.float32(0), r).astype(np.float32)


def _uniform(rng, shape, bound):
    return rng.uniform(-bound, bound, size=shape).astype(np.float32)


# --------------------------------------------------------------------------------------
# Weights (reading S25): W ~ U(+-scale/sqrt(h)), bias ~ U(+-1/sqrt(h)), E ~ N(0, 1).
# All layouts are the "paper/oracle" layouts documented in include/bm.h:
#   LSTM layer  W [4h, 2h] row-major, columns = [x ; h], gate row blocks (i, f, g, o)
#   tree leaf   W [3h,  h], gate row blocks (i, o, u)
#   tree intern U [5h, 2h], columns = [h_L ; h_R], gate row blocks (i, f_L, f_R, o, u)
#   embedding   E [V, h];  output projection W_out [V, h], b_out [V]
# --------------------------------------------------------------------------------------

@dataclasses.dataclass
class LSTMStackWeights:
    hidden: int
    vocab: int
    W: List[np.ndarray]        # per layer [4h, 2h] fp32
    b: List[np.ndarray]        # per layer [4h] fp32
    E: np.ndarray              # [V, h] fp32
    W_out: Optional[np.ndarray] = None   # [V, h] (decoder only)
    b_out: Optional[np.ndarray] = None   # [V]

    @property
    def layers(self) -> int:
        return len(self.W)


@dataclasses.dataclass
class TreeWeights:
    hidden: int
    vocab: int
    W_leaf: np.ndarray   # [3h, h]
    b_leaf: np.ndarray   # [3h]
    U: np.ndarray        # [5h, 2h]
    b_int: np.ndarray    # [5h]
    E: np.ndarray        # [V, h]


def lstm_stack_weights(hidden: int, layers: int, vocab: int, seed: int, scale: float = 2.0,
                       projection: bool = False, bf16: bool = True) -> LSTMStackWeights:
    rng = np.random.default_rng(seed)
    h = hidden
    rnd = bf16_round if bf16 else (lambda a: a.astype(np.float32))
    W = [rnd(_uniform(rng, (4 * h, 2 * h), scale / np.sqrt(h))) for _ in range(layers)]
    b = [rnd(_uniform(rng, (4 * h,), 1.0 / np.sqrt(h))) for _ in range(layers)]
    E = rnd(rng.standard_normal((vocab, h)).astype(np.float32))
    W_out = b_out = None
    if projection:
        W_out = rnd(_uniform(rng, (vocab, h), scale / np.sqrt(h)))
        b_out = rnd(_uniform(rng, (vocab,), 1.0 / np.sqrt(h)))
    return LSTMStackWeights(h, vocab, W, b, E, W_out, b_out)


def tree_weights(hidden: int, vocab: int, seed: int, scale: float = 2.0,
                 bf16: bool = True) -> TreeWeights:
    rng = np.random.default_rng(seed)
    h = hidden
    rnd = bf16_round if bf16 else (lambda a: a.astype(np.float32))
    W_leaf = rnd(_uniform(rng, (3 * h, h), scale / np.sqrt(h)))
    b_leaf = rnd(_uniform(rng, (3 * h,), 1.0 / np.sqrt(h)))
    U = rnd(_uniform(rng, (5 * h, 2 * h), scale / np.sqrt(h)))
    b_int = rnd(_uniform(rng, (5 * h,), 1.0 / np.sqrt(h)))
    E = rnd(rng.standard_normal((vocab, h)).astype(np.float32))
    return TreeWeights(h, vocab, W_leaf, b_leaf, U, b_int, E)


# --------------------------------------------------------------------------------------
# Requests
# --------------------------------------------------------------------------------------

@dataclasses.dataclass
class Request:
    """One inference request as submitted (mirrors bm_request in include/bm.h).

    kind CHAIN:   tokens[L]                     (one LSTM cell type)
    kind SEQ2SEQ: tokens[S_src] source, decode_len T (decoder runs exactly T steps, L715)
    kind TREE:    n_nodes in post-order, root last; left/right child index or -1;
                  tokens[n] (word id at leaves, ignored at internal nodes)
    arrival: virtual tick (virtual-time mode) or seconds (wall-clock mode)."""
    kind: int
    tokens: np.ndarray
    arrival: float = 0.0
    decode_len: int = 0
    left: Optional[np.ndarray] = None
    right: Optional[np.ndarray] = None

    @property
    def length(self) -> int:
        return int(len(self.tokens))


def wmt_lengths(n: int, rng: np.random.Generator) -> np.ndarray:
    """Sentence lengths shaped like WMT-15 Europarl (L421, L635; reading in SURVEY §8d):
    clip(round(lognormal(mu=2.914, sigma=0.727)), 1, 330) -> mean ~24, median ~18, p99 ~100."""
    return np.clip(np.round(rng.lognormal(2.914, 0.727, size=n)), 1, 330).astype(np.int64)


def poisson_arrivals(n: int, rate: float, rng: np.random.Generator, start: float = 0.0) -> np.ndarray:
    """Open-loop Poisson arrivals (exponential gaps) at `rate` requests per time unit (L423)."""
    gaps = rng.exponential(1.0 / rate, size=n)
    return start + np.cumsum(gaps) - gaps[0]


def _tokens(rng, n, vocab):
    return rng.integers(FIRST_PAYLOAD, vocab, size=n).astype(np.int32)


def chain_trace(n: int, vocab: int, seed: int, rate: Optional[float] = None,
                lengths: Optional[Sequence[int]] = None,
                arrivals: Optional[Sequence[float]] = None) -> List[Request]:
    rng = np.random.default_rng(seed)
    L = np.asarray(lengths if lengths is not None else wmt_lengths(n, rng))
    if arrivals is None:
        arrivals = poisson_arrivals(n, rate, rng) if rate else np.zeros(n)
    return [Request(CHAIN, _tokens(rng, int(L[i]), vocab), float(arrivals[i])) for i in range(n)]


def seq2seq_trace(n: int, vocab: int, seed: int, rate: Optional[float] = None,
                  max_len: int = 330) -> List[Request]:
    """Source lengths WMT-like; target length = clip(round(src * exp(N(0, 0.2))), 1, 330)."""
    rng = np.random.default_rng(seed)
    src = np.minimum(wmt_lengths(n, rng), max_len)
    tgt = np.clip(np.round(src * np.exp(rng.normal(0.0, 0.2, size=n))), 1, max_len).astype(np.int64)
    arrivals = poisson_arrivals(n, rate, rng) if rate else np.zeros(n)
    return [Request(SEQ2SEQ, _tokens(rng, int(src[i]), vocab), float(arrivals[i]),
                    decode_len=int(tgt[i])) for i in range(n)]


def _random_bracketing(n_leaves: int, rng: np.random.Generator):
    """Binary tree over n_leaves leaves by recursive uniform split point; returns
    post-order (left, right) child arrays with -1 for leaves."""
    left: List[int] = []
    right: List[int] = []

    def build(lo: int, hi: int) -> int:   # leaves [lo, hi)
        if hi - lo == 1:
            left.append(-1)
            right.append(-1)
            return len(left) - 1
        split = int(rng.integers(lo + 1, hi))
        l = build(lo, split)
        r = build(split, hi)
        left.append(l)
        right.append(r)
        return len(left) - 1

    build(0, n_leaves)
    return np.asarray(left, np.int32), np.asarray(right, np.int32)


def complete_tree(n_leaves: int = 16):
    """Complete binary tree in post-order (the identical-tree workload of L857)."""
    assert n_leaves & (n_leaves - 1) == 0
    left: List[int] = []
    right: List[int] = []

    def build(size: int) -> int:
        if size == 1:
            left.append(-1)
            right.append(-1)
            return len(left) - 1
        l = build(size // 2)
        r = build(size // 2)
        left.append(l)
        right.append(r)
        return len(left) - 1

    build(n_leaves)
    return np.asarray(left, np.int32), np.asarray(right, np.int32)


def treebank_leaves(n: int, rng: np.random.Generator) -> np.ndarray:
    """Leaf counts shaped like Stanford TreeBank sentences (reading S26):
    clip(round(lognormal(ln 18, 0.5)), 2, 56)."""
    return np.clip(np.round(rng.lognormal(np.log(18.0), 0.5, size=n)), 2, 56).astype(np.int64)


def tree_trace(n: int, vocab: int, seed: int, rate: Optional[float] = None,
               identical: bool = False, n_leaves: Optional[Sequence[int]] = None) -> List[Request]:
    rng = np.random.default_rng(seed)
    leaves = treebank_leaves(n, rng) if n_leaves is None else np.asarray(n_leaves)
    arrivals = poisson_arrivals(n, rate, rng) if rate else np.zeros(n)
    out = []
    for i in range(n):
        if identical:
            left, right = complete_tree(16)
        else:
            left, right = _random_bracketing(int(leaves[i]), rng)
        toks = _tokens(rng, len(left), vocab)
        toks[left >= 0] = PAD
        out.append(Request(TREE, toks, float(arrivals[i]), left=left, right=right))
    return out


# --------------------------------------------------------------------------------------
# Fixed fixtures
# --------------------------------------------------------------------------------------

def figure5_trace(vocab: int = 128, seed: int = 5) -> List[Request]:
    """Figure 5 (L223-L271): eight chain requests, lengths 2,3,3,5 at t=0 and 5,7,3,1
    arriving later. The paper does not print the later arrival ticks; the reading used
     is req5@1, req6@2, req7@2, req8@4."""
    return chain_trace(8, vocab, seed, lengths=[2, 3, 3, 5, 5, 7, 3, 1],
                       arrivals=[0, 0, 0, 0, 1, 2, 2, 4])


def config0_trace(vocab: int = 128, seed: int = 0) -> List[Request]:
    """BASELINE configs[0]: 4 requests, lengths (3, 10, 5, 8), arrivals (0, 0, 1, 3)."""
    return chain_trace(4, vocab, seed, lengths=[3, 10, 5, 8], arrivals=[0, 0, 1, 3])
