"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu).

bench.py's own engine builder, weights and trace generator are used unchanged: configs[1]
(20 000 WMT-length requests, h = 1024, V = 32768, bmax 512, 65 536 pool slots, look-ahead 2,
wall clock, open-loop Poisson arrivals at a saturating rate, so tasks span the single-CTA and
the CTA-pair kernels), configs[3] (6 000 TreeBank-shaped trees, bmax 64) and configs[2]
(Seq2Seq 4+4 layers, encoder/decoder bmax 512/256). Every request must complete; a seeded
sample of requests is recomputed one by one by the fp64 oracle (forced-token mode for the
decoder) and compared at north_star's bf16 tolerance."""
import numpy as np
import pytest

import bench
from gpu_helpers import TOL
from oracle import cells
from paper_conf_eurosys_gaoywl18_b200 import bm
from workloads import gen

pytestmark = pytest.mark.gpu


def _run_bench_config(wl, n, rate, seed=1000):
    w = bench.make_weights(wl)
    e, cellmap = bench.build_engine(bm, wl, w, 0, max_requests=n + 64, lookahead=bench.WL[wl]["lookahead"],
                                    time_kernels=0, keep=1)
    trace = bench.make_trace(wl, n, rate, seed)
    prep = e.prepare_requests(trace, cellmap)
    first = e.submit_many(prep)
    assert e.run() == n
    comp = e.poll(n + 16)
    assert sorted(c.req_id for c in comp) == list(range(first, first + n))
    return e, w, trace, first


def test_configs1_full_size_sampled():
    n = bench.WL["lstm"]["reqs"]
    e, w, trace, first = _run_bench_config("lstm", n, rate=650000.0)
    rng = np.random.default_rng(7)
    sample = np.concatenate([[0, n - 1], rng.choice(n, 14, replace=False),
                             [int(np.argmax([len(q.tokens) for q in trace]))]])  # longest request too
    worst = 0.0
    for i in sample:
        r = e.read_result(first + int(i), 1)
        hs, cs = cells.chain_lstm(w["cell"], trace[i].tokens)
        worst = max(worst, np.max(np.abs(r["h"][0] - hs[0])), np.max(np.abs(r["c"][0] - cs[0])))
    assert worst <= TOL[bm.PREC_BF16], worst
    e.close()


def test_configs3_full_size_sampled():
    n = bench.WL["tree"]["reqs"]
    e, w, trace, first = _run_bench_config("tree", n, rate=60000.0)
    rng = np.random.default_rng(8)
    worst = 0.0
    for i in np.concatenate([[0, n - 1], rng.choice(n, 30, replace=False)]):
        q = trace[int(i)]
        r = e.read_result(first + int(i), 1)
        rh, rc, _ = cells.tree_lstm(w["tree"], q.tokens, q.left, q.right)
        worst = max(worst, np.max(np.abs(r["h"][0] - rh)), np.max(np.abs(r["c"][0] - rc)))
    assert worst <= TOL[bm.PREC_BF16], worst
    e.close()


def test_configs2_full_size_sampled():
    n = 1000  # of bench.WL["seq2seq"]["reqs"] = 4000: same engine, same generator, same rate regime
    e, w, trace, first = _run_bench_config("seq2seq", n, rate=20000.0)
    L = bench.WL["seq2seq"]["layers"]
    tol = TOL[bm.PREC_BF16]
    rng = np.random.default_rng(9)
    for i in np.concatenate([[0], rng.choice(n, 3, replace=False)]):
        q = trace[int(i)]
        r = e.read_result(first + int(i), L, decode_len=q.decode_len)
        o = cells.seq2seq(w["enc"], w["dec"], q.tokens, q.decode_len, forced_tokens=r["tokens"])
        for s in range(q.decode_len):
            assert o["logits"][s][r["tokens"][s]] >= o["logits"][s].max() - 2 * tol
        for l in range(L):
            assert np.max(np.abs(r["h"][l] - o["h"][l])) <= tol
            assert np.max(np.abs(r["c"][l] - o["c"][l])) <= tol
    e.close()
