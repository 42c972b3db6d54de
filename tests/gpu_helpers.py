"""Shared helpers for the -m gpu parity tests: build engines with the seeded weights of
workloads.gen and run the oracle on exactly the inputs the device sees."""
import numpy as np

from paper_conf_eurosys_gaoywl18_b200 import bm
from workloads import gen

TOL = {bm.PREC_BF16: 5e-3, bm.PREC_FP32: 1e-5}   # north_star tolerances


def lstm_engine(h, layers, vocab, prec, bmax=512, seed=0, clock=bm.CLOCK_WALL, proj=False,
                max_slots=4096, max_requests=4096, **kw):
    w = gen.lstm_stack_weights(h, layers, vocab, seed, projection=proj, bf16=(prec == bm.PREC_BF16))
    e = bm.Engine(precision=prec, clock=clock, hidden=h, pool_layers=layers, max_slots=max_slots,
                  max_requests=max_requests, **kw)
    kind = bm.CELL_LSTM_PROJ if proj else bm.CELL_LSTM
    cid = e.load_cell(kind, layers, vocab, bmax, 1 if proj else 0, w.W, w.b, w.E, w.W_out, w.b_out)
    return e, cid, w


def seq2seq_engine(h, layers, vocab, prec, bmax=(512, 256), seed=0, clock=bm.CLOCK_WALL, **kw):
    bf = prec == bm.PREC_BF16
    enc = gen.lstm_stack_weights(h, layers, vocab, seed, bf16=bf)
    dec = gen.lstm_stack_weights(h, layers, vocab, seed + 1, projection=True, bf16=bf)
    e = bm.Engine(precision=prec, clock=clock, hidden=h, pool_layers=layers, **kw)
    ce = e.load_cell(bm.CELL_LSTM, layers, vocab, bmax[0], 0, enc.W, enc.b, enc.E)
    cd = e.load_cell(bm.CELL_LSTM_PROJ, layers, vocab, bmax[1], 1, dec.W, dec.b, dec.E, dec.W_out, dec.b_out)
    return e, (ce, cd), (enc, dec)


def tree_engine(h, vocab, prec, bmax=64, seed=0, clock=bm.CLOCK_WALL, **kw):
    w = gen.tree_weights(h, vocab, seed, bf16=(prec == bm.PREC_BF16))
    e = bm.Engine(precision=prec, clock=clock, hidden=h, pool_layers=1, **kw)
    leaf = e.load_cell(bm.CELL_TREE_LEAF, 1, vocab, bmax, 0, [w.W_leaf], [w.b_leaf], w.E)
    intern = e.load_cell(bm.CELL_TREE_INTERNAL, 1, vocab, bmax, 1, [w.U], [w.b_int])
    return e, (leaf, intern), w


def bf16_vals(x, prec):
    return gen.bf16_round(np.asarray(x, np.float32)) if prec == bm.PREC_BF16 else np.asarray(x, np.float32)
