"""Small workloads for compute-sanitizer memcheck (tools/sanitize.sh): configs[0] (h=64) and a
few h=1024 chain requests through the C-ABI engine, plus one h=64 Seq2Seq and one small tree."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_gaoywl18_b200 import bm  # noqa: E402
from workloads import gen  # noqa: E402

w = gen.lstm_stack_weights(64, 1, 128, seed=0)
e = bm.Engine(clock=bm.CLOCK_VIRTUAL, hidden=64, max_slots=16, max_requests=16, keep_results=1)
cid = e.load_cell(bm.CELL_LSTM, 1, 128, 4, 0, w.W, w.b, w.E)
for q in gen.config0_trace(vocab=128):
    e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
assert e.run() == 4
e.close()
w = gen.lstm_stack_weights(1024, 1, 512, seed=0)
e = bm.Engine(clock=bm.CLOCK_VIRTUAL, hidden=1024, max_slots=64, max_requests=64, keep_results=1,
              schedule_when_outstanding_leq=2)
cid = e.load_cell(bm.CELL_LSTM, 1, 512, 512, 0, w.W, w.b, w.E)
for q in gen.chain_trace(12, 512, seed=3, rate=4.0):
    e.submit(bm.REQ_CHAIN, cid, 0, q.tokens, q.arrival)
assert e.run() == 12
e.close()
enc = gen.lstm_stack_weights(64, 2, 256, seed=0)
dec = gen.lstm_stack_weights(64, 2, 256, seed=1, projection=True)
e = bm.Engine(clock=bm.CLOCK_VIRTUAL, hidden=64, pool_layers=2, max_slots=8, max_requests=8, keep_results=1,
              max_decode_len=8)
ce = e.load_cell(bm.CELL_LSTM, 2, 256, 512, 0, enc.W, enc.b, enc.E)
cd = e.load_cell(bm.CELL_LSTM_PROJ, 2, 256, 256, 1, dec.W, dec.b, dec.E, dec.W_out, dec.b_out)
e.submit(bm.REQ_SEQ2SEQ, ce, cd, np.array([5, 9, 77], np.int32), 0, decode_len=5, eos_id=3)
assert e.run() == 1
e.close()
tw = gen.tree_weights(64, 100, seed=0)
e = bm.Engine(clock=bm.CLOCK_VIRTUAL, hidden=64, max_slots=64, max_requests=4, keep_results=1)
leaf = e.load_cell(bm.CELL_TREE_LEAF, 1, 100, 64, 0, [tw.W_leaf], [tw.b_leaf], tw.E)
intern = e.load_cell(bm.CELL_TREE_INTERNAL, 1, 100, 64, 1, [tw.U], [tw.b_int])
left, right = gen.complete_tree(8)
toks = np.where(left < 0, np.arange(len(left)) + 3, 0).astype(np.int32)
e.submit(bm.REQ_TREE, leaf, intern, toks, 0, left=left, right=right)
assert e.run() == 1
e.close()
print("memcheck workload ok")
