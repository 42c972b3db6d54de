"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu).

bench.py's own engine builder, weights and trace generator are used unchanged: configs[1]
(20 000 WMT-length requests, h = 1024, V = 32768, bmax 512, 65 536 pool slots, look-ahead 2,
wall clock, open-loop Poisson arrivals at a saturating rate, so tasks span the single-CTA and
the CTA-pair kernels), configs[3] (6 000 TreeBank-shaped trees, bmax 64) and configs[2]
(4 000 Seq2Seq requests, 4+4 layers, encoder/decoder bmax 512/256). Every request must
complete and EVERY request's result is compared with the fp64 oracle: the oracle's batched
executors (oracle/batched.py, pinned row for row against the unbatched oracle by
tests/test_oracle_batching.py; batching only concatenates independent rows, §3.1) run
all requests in lockstep on the host cores. The decoder runs in forced-token mode (SURVEY
§8c): every emitted token must be a valid argmax of the fp64 logits within 2 tol, and the
final per-layer h, c of every request must agree within north_star's bf16 tolerance."""
import numpy as np
import pytest

import bench
from gpu_helpers import TOL
from oracle import batched
from paper_conf_eurosys_gaoywl18_b200 import bm

pytestmark = pytest.mark.gpu


def _blas_threads():
    try:
        from threadpoolctl import threadpool_limits
        import os
        return threadpool_limits(limits=os.cpu_count() or 1)
    except Exception:  # pragma: no cover
        import contextlib
        return contextlib.nullcontext()


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
    L, H = bench.WL[wl]["layers"], bench.WL[wl]["hidden"]
    hh = np.zeros((n, L, H), np.float32)
    cc = np.zeros((n, L, H), np.float32)
    toks = np.zeros((n, 340), np.int32) if wl == "seq2seq" else None
    e.read_results_many(first, n, h=hh, c=cc, tokens=toks, release=False)
    e.close()
    return w, trace, hh, cc, toks


def test_configs1_full_size_every_request():
    n = bench.WL["lstm"]["reqs"]
    w, trace, hh, cc, _ = _run_bench_config("lstm", n, rate=650000.0)
    toks = [q.tokens for q in trace]
    steps = max(len(t) for t in toks)
    sched = [[(r, k) for r in range(n) if len(toks[r]) > k] for k in range(steps)]
    with _blas_threads():
        ref = batched.run_chain_schedule(w["cell"], toks, sched)
    err_h = np.array([np.max(np.abs(hh[r, 0] - ref[r][0][0])) for r in range(n)])
    err_c = np.array([np.max(np.abs(cc[r, 0] - ref[r][1][0])) for r in range(n)])
    assert err_h.max() <= TOL[bm.PREC_BF16], (int(err_h.argmax()), err_h.max())
    assert err_c.max() <= TOL[bm.PREC_BF16], (int(err_c.argmax()), err_c.max())


def _heights(left, right):
    ht = np.zeros(len(left), np.int64)
    for v in range(len(left)):
        if left[v] >= 0:
            ht[v] = 1 + max(ht[left[v]], ht[right[v]])
    return ht


def test_configs3_full_size_every_request():
    n = bench.WL["tree"]["reqs"]
    w, trace, hh, cc, _ = _run_bench_config("tree", n, rate=60000.0)
    trees = [(q.tokens, q.left, q.right) for q in trace]
    hts = [_heights(q.left, q.right) for q in trace]
    top = max(int(h.max()) for h in hts)
    # level by level: all leaves, then every internal node of height 1, 2, ... (a valid
    # dependency-respecting schedule; the leaf and internal cell types never share a task)
    sched = [[(t, v) for t in range(n) for v in np.flatnonzero(hts[t] == k)] for k in range(top + 1)]
    with _blas_threads():
        ref = batched.run_tree_schedule(w["tree"], trees, sched)
    err = max(max(np.max(np.abs(hh[t, 0] - ref[t][0])), np.max(np.abs(cc[t, 0] - ref[t][1])))
              for t in range(n))
    assert err <= TOL[bm.PREC_BF16], err


def test_configs2_full_size_every_request():
    n = bench.WL["seq2seq"]["reqs"]
    w, trace, hh, cc, toks = _run_bench_config("seq2seq", n, rate=20000.0)
    L = bench.WL["seq2seq"]["layers"]
    tol = TOL[bm.PREC_BF16]
    forced = [toks[r, :trace[r].decode_len] for r in range(n)]
    assert all((f >= 0).all() for f in forced)
    with _blas_threads():
        H_, C_, sel, best = batched.run_seq2seq_forced_lockstep(w["enc"], w["dec"], [q.tokens for q in trace],
                                                                forced)
    gap = max(float(np.max(best[r] - sel[r])) for r in range(n))
    assert gap <= 2 * tol, gap   # every emitted token a valid argmax within 2 tol
    errs = np.array([[max(np.max(np.abs(hh[r, l] - H_[r][l])), np.max(np.abs(cc[r, l] - C_[r][l])))
                      for l in range(L)] for r in range(n)])
    r = int(errs.max(1).argmax())
    assert errs.max() <= tol, {"req": r, "src": len(trace[r].tokens), "tgt": trace[r].decode_len,
                               "err_by_layer": errs[r].tolist(), "n_over": int((errs.max(1) > tol).sum())}
