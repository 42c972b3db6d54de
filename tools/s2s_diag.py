"""Diagnose the configs[2] full-size parity gap: per-request error of the device against the
fp64 oracle (batched lockstep, forced tokens), by layer and by length; and, for the worst
requests, the error against a bf16-ACTIVATION emulation (fp64 arithmetic, h rounded to bf16 after
every step as the pool stores it) -- if the device matches the emulation closely while both
differ from the oracle, the gap is the precision of bf16 activations over long recurrences, not
a kernel fault. Tool only (not a test, not an oracle)."""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import bench  # noqa: E402
from oracle import batched  # noqa: E402
from paper_conf_eurosys_gaoywl18_b200 import bm  # noqa: E402
from workloads import gen  # noqa: E402


def bf16(x):
    return gen.bf16_round(np.asarray(x, np.float32)).astype(np.float64)


def emulate(enc, dec, src, forced):
    """fp64 recurrence with every stored h rounded to bf16 (the device pool's storage)."""
    from oracle.cells import GO, sigmoid
    L, H = enc.layers, enc.hidden
    h = [np.zeros(H) for _ in range(L)]
    c = [np.zeros(H) for _ in range(L)]

    def step(w, x):
        for l in range(L):
            z = w.W[l].astype(np.float64) @ np.concatenate([x, h[l]]) + w.b[l]
            i, f = sigmoid(z[:H]), sigmoid(z[H:2 * H])
            g, o = np.tanh(z[2 * H:3 * H]), sigmoid(z[3 * H:])
            c[l] = f * c[l] + i * g
            h[l] = bf16(o * np.tanh(c[l]))
            x = h[l]
    for t in src:
        step(enc, enc.E[int(t)].astype(np.float64))
    prev = GO
    for s in range(len(forced)):
        step(dec, dec.E[prev].astype(np.float64))
        prev = int(forced[s])
    return h, c


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 4000
    from threadpoolctl import threadpool_limits
    w = bench.make_weights("seq2seq")
    e, cellmap = bench.build_engine(bm, "seq2seq", w, 0, max_requests=n + 64, lookahead=1, time_kernels=0, keep=1)
    trace = bench.make_trace("seq2seq", n, 20000.0, 1000)
    prep = e.prepare_requests(trace, cellmap)
    first = e.submit_many(prep)
    assert e.run() == n
    e.poll(n + 16)
    L, H = 4, 1024
    hh = np.zeros((n, L, H), np.float32)
    cc = np.zeros((n, L, H), np.float32)
    toks = np.zeros((n, 340), np.int32)
    e.read_results_many(first, n, h=hh, c=cc, tokens=toks, release=False)
    forced = [toks[r, :trace[r].decode_len] for r in range(n)]
    with threadpool_limits(limits=os.cpu_count()):
        H_, C_, sel, best = batched.run_seq2seq_forced_lockstep(w["enc"], w["dec"], [q.tokens for q in trace], forced)
    eh = np.array([[np.max(np.abs(hh[r, l] - H_[r][l])) for l in range(L)] for r in range(n)])
    ec = np.array([[np.max(np.abs(cc[r, l] - C_[r][l])) for l in range(L)] for r in range(n)])
    err = np.maximum(eh.max(1), ec.max(1))
    src = np.array([len(q.tokens) for q in trace])
    tgt = np.array([q.decode_len for q in trace])
    out = {"n": n, "max_err": float(err.max()), "frac_over_5e-3": float((err > 5e-3).mean()),
           "quantiles": {q: float(np.quantile(err, q)) for q in (0.5, 0.9, 0.99, 0.999)},
           "err_by_total_len": {}}
    tot = src + tgt
    for lo, hi in ((1, 25), (25, 50), (50, 100), (100, 200), (200, 700)):
        m = (tot >= lo) & (tot < hi)
        if m.any():
            out["err_by_total_len"][f"{lo}-{hi}"] = {"n": int(m.sum()), "max": float(err[m].max()),
                                                     "p99": float(np.quantile(err[m], 0.99))}
    worst = np.argsort(-err)[:4]
    rows = []
    for r in worst:
        with threadpool_limits(limits=os.cpu_count()):
            eh_, ec_ = emulate(w["enc"], w["dec"], trace[r].tokens, forced[r])
        rows.append({"req": int(r), "src": int(src[r]), "tgt": int(tgt[r]), "err_vs_oracle": float(err[r]),
                     "err_h_by_layer": eh[r].round(5).tolist(), "err_c_by_layer": ec[r].round(5).tolist(),
                     "device_vs_bf16_emulation": float(max(max(np.max(np.abs(hh[r, l] - eh_[l])) for l in range(L)),
                                                           max(np.max(np.abs(cc[r, l] - ec_[l])) for l in range(L)))),
                     "oracle_vs_bf16_emulation": float(max(max(np.max(np.abs(H_[r][l] - eh_[l])) for l in range(L)),
                                                           max(np.max(np.abs(C_[r][l] - ec_[l])) for l in range(L))))})
    out["worst"] = rows
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
