"""Pins for the fp64 oracle: the oracle is checked against things other
than itself — a closed form, an independent library implementation (torch.nn.LSTMCell /
nn.LSTM in float64) and structural reductions/invariants of the TreeLSTM."""
import numpy as np
import pytest
import torch

from oracle import cells
from workloads import gen


def _w(h=8, layers=1, vocab=16, seed=0, projection=False):
    return gen.lstm_stack_weights(h, layers, vocab, seed, projection=projection, bf16=False)


# ----------------------------------------------------------------------------- P1
@pytest.mark.parametrize("beta", [0.375, -1.125, 2.0])  # exact in fp32
@pytest.mark.parametrize("layers", [1, 4])
def test_p1_closed_form(beta, layers):
    """Zero W and bias except the g-bias beta: i = f = o = 1/2, g = tanh(beta), so
    c_t = tanh(beta) (1 - 2^-t) and h_t = tanh(c_t) / 2 in every layer (footnote 2 L205
    shapes; standard LSTM equations, reading S1)."""
    h = 8
    w = _w(h, layers)
    for l in range(layers):
        w.W[l][:] = 0
        w.b[l][:] = 0
        w.b[l][2 * h:3 * h] = beta
    for t in range(1, 12):
        hs, cs = cells.chain_lstm(w, [3] * t)
        c_exp = np.tanh(beta) * (1 - 2.0 ** -t)
        for l in range(layers):
            np.testing.assert_allclose(cs[l], c_exp, rtol=0, atol=2e-16)
            np.testing.assert_allclose(hs[l], 0.5 * np.tanh(c_exp), rtol=0, atol=2e-16)


# ----------------------------------------------------------------------------- P2
def _torch_cell(w, l):
    h = w.hidden
    cell = torch.nn.LSTMCell(h, h, dtype=torch.float64)
    with torch.no_grad():
        W = torch.from_numpy(w.W[l].astype(np.float64))
        cell.weight_ih.copy_(W[:, :h])   # torch gate layout of weight_ih: (i, f, g, o)
        cell.weight_hh.copy_(W[:, h:])
        cell.bias_ih.copy_(torch.from_numpy(w.b[l].astype(np.float64)))
        cell.bias_hh.zero_()
    return cell


@pytest.mark.parametrize("h", [1, 8, 64])
def test_p2_lstm_cell_vs_torch(h):
    w = _w(h, 1, vocab=32, seed=h)
    toks = [5, 9, 3, 31, 7, 7, 12]
    hs, cs = cells.chain_lstm(w, toks)
    cell = _torch_cell(w, 0)
    th = torch.zeros(1, h, dtype=torch.float64)
    tc = torch.zeros(1, h, dtype=torch.float64)
    with torch.no_grad():
        for t in toks:
            th, tc = cell(torch.from_numpy(w.E[t].astype(np.float64))[None], (th, tc))
    np.testing.assert_allclose(hs[0], th[0].numpy(), rtol=0, atol=1e-14)
    np.testing.assert_allclose(cs[0], tc[0].numpy(), rtol=0, atol=1e-14)


def _torch_stack(w):
    h, L = w.hidden, w.layers
    m = torch.nn.LSTM(h, h, num_layers=L, dtype=torch.float64)
    with torch.no_grad():
        for l in range(L):
            W = torch.from_numpy(w.W[l].astype(np.float64))
            getattr(m, f"weight_ih_l{l}").copy_(W[:, :h])
            getattr(m, f"weight_hh_l{l}").copy_(W[:, h:])
            getattr(m, f"bias_ih_l{l}").copy_(torch.from_numpy(w.b[l].astype(np.float64)))
            getattr(m, f"bias_hh_l{l}").zero_()
    return m


def test_p2_stack_vs_torch_lstm():
    w = _w(16, 4, vocab=40, seed=3)
    toks = [4, 8, 15, 16, 23, 39]
    hs, cs = cells.chain_lstm(w, toks)
    m = _torch_stack(w)
    x = torch.from_numpy(w.E[toks].astype(np.float64))[:, None, :]
    with torch.no_grad():
        _, (hn, cn) = m(x)
    for l in range(4):
        np.testing.assert_allclose(hs[l], hn[l, 0].numpy(), rtol=0, atol=1e-14)
        np.testing.assert_allclose(cs[l], cn[l, 0].numpy(), rtol=0, atol=1e-14)


def test_p2_seq2seq_vs_torch():
    """Encoder = nn.LSTM over E_src; decoder = same stack stepped with feed-previous from
    <go>, logits = F.linear(h_L, W_out, b_out), y = torch.argmax (first maximal index)."""
    h, L, V = 16, 4, 50
    enc = _w(h, L, V, seed=10)
    dec = _w(h, L, V, seed=11, projection=True)
    src = [7, 3, 44, 12]
    T = 6
    out = cells.seq2seq(enc, dec, src, T)
    me, md = _torch_stack(enc), _torch_stack(dec)
    with torch.no_grad():
        _, (hn, cn) = me(torch.from_numpy(enc.E[src].astype(np.float64))[:, None, :])
        prev = gen.GO
        toks, logits = [], []
        for _ in range(T):
            x = torch.from_numpy(dec.E[prev].astype(np.float64))[None, None, :]
            y, (hn, cn) = md(x, (hn, cn))
            lg = torch.nn.functional.linear(y[0, 0], torch.from_numpy(dec.W_out.astype(np.float64)),
                                            torch.from_numpy(dec.b_out.astype(np.float64)))
            prev = int(torch.argmax(lg))
            toks.append(prev)
            logits.append(lg.numpy())
    assert out["tokens"] == toks
    np.testing.assert_allclose(out["logits"], np.array(logits), rtol=0, atol=1e-13)
    for l in range(L):
        np.testing.assert_allclose(out["h"][l], hn[l, 0].numpy(), rtol=0, atol=1e-14)
        np.testing.assert_allclose(out["c"][l], cn[l, 0].numpy(), rtol=0, atol=1e-14)


def test_argmax_lowest_index_on_ties():
    assert cells.argmax_lowest(np.array([0.0, 2.0, 1.0, 2.0])) == 1
    assert cells.argmax_lowest(np.array([5.0, 5.0])) == 0


def test_seq2seq_forced_tokens_follow_given_sequence():
    h, L, V = 8, 2, 20
    enc, dec = _w(h, L, V, seed=1), _w(h, L, V, seed=2, projection=True)
    forced = [5, 6, 7]
    out = cells.seq2seq(enc, dec, [4, 9], 3, forced_tokens=forced)
    assert out["fed_tokens"] == forced
    # the decoder input at step s is E[forced[s-1]]: re-running free with the same first
    # argmax must agree on step 0 logits
    free = cells.seq2seq(enc, dec, [4, 9], 1)
    np.testing.assert_array_equal(out["logits"][0], free["logits"][0])


def _torch_decode_forced(enc, dec, src, fed):
    """Independent decoder (P2 library routine): encoder = nn.LSTM over E_src; decoder step s
    = nn.LSTM stepped on E_tgt[<go>] at s = 0 and on E_tgt[fed[s-1]] after (feed-previous
    with the given tokens, L713-L715); logits = F.linear(h_L, W_out, b_out)."""
    me, md = _torch_stack(enc), _torch_stack(dec)
    Wo = torch.from_numpy(dec.W_out.astype(np.float64))
    bo = torch.from_numpy(dec.b_out.astype(np.float64))
    out = []
    with torch.no_grad():
        _, (hn, cn) = me(torch.from_numpy(enc.E[src].astype(np.float64))[:, None, :])
        prev = gen.GO
        for s in range(len(fed)):
            y, (hn, cn) = md(torch.from_numpy(dec.E[prev].astype(np.float64))[None, None, :], (hn, cn))
            out.append(torch.nn.functional.linear(y[0, 0], Wo, bo).numpy())
            prev = int(fed[s])
    return np.array(out), hn, cn


@pytest.mark.parametrize("k", [0, 2, 4])
def test_p2_seq2seq_forced_token_mode_vs_torch(k):
    """Forced-token mode (decoding per L715) pinned against an independent decoder:
    take the free run's tokens and change the one emitted at step k. Then (i) the logits of
    steps <= k are exactly the free run's (the change only reaches the input of step k+1),
    (ii) every step's logits and the final per-layer (h, c) equal torch nn.LSTM stepped on the
    forced tokens, and (iii) step k+1 differs from the free run (the forced token was fed,
    not the oracle's own argmax). A decoder that feeds its own argmax fails (ii)."""
    h, L, V, T = 16, 4, 50, 6
    enc = _w(h, L, V, seed=20)
    dec = _w(h, L, V, seed=21, projection=True)
    src = [9, 31, 4, 17, 40]
    free = cells.seq2seq(enc, dec, src, T)
    forced = list(free["tokens"])
    forced[k] = (forced[k] + 7) % V
    out = cells.seq2seq(enc, dec, src, T, forced_tokens=forced)
    np.testing.assert_array_equal(out["logits"][:k + 1], free["logits"][:k + 1])
    ref, hn, cn = _torch_decode_forced(enc, dec, src, forced)
    np.testing.assert_allclose(out["logits"], ref, rtol=0, atol=1e-13)
    for l in range(L):
        np.testing.assert_allclose(out["h"][l], hn[l, 0].numpy(), rtol=0, atol=1e-14)
        np.testing.assert_allclose(out["c"][l], cn[l, 0].numpy(), rtol=0, atol=1e-14)
    assert np.max(np.abs(out["logits"][k + 1] - free["logits"][k + 1])) > 1e-6
    # the oracle's own argmax is still reported for the validity check
    assert out["tokens"] == [cells.argmax_lowest(z) for z in out["logits"]]


def test_seq2seq_forced_tokens_terminate_at_forced_eos():
    """With eos_stop, termination follows the FED token (N1 under forced-token mode): forcing
    the eos id at step k ends decoding after step k; the state then equals torch's after k+1
    steps."""
    h, L, V, T, k = 16, 2, 40, 8, 3
    enc = _w(h, L, V, seed=22)
    dec = _w(h, L, V, seed=23, projection=True)
    src = [5, 6, 7]
    free = cells.seq2seq(enc, dec, src, T)
    eos = (free["tokens"][k] + 1) % V
    forced = [t if t != eos else (t + 2) % V for t in free["tokens"]]
    forced[k] = eos
    out = cells.seq2seq(enc, dec, src, T, forced_tokens=forced, eos_id=eos)
    assert len(out["logits"]) == k + 1 and out["fed_tokens"][-1] == eos
    ref, hn, cn = _torch_decode_forced(enc, dec, src, forced[:k + 1])
    np.testing.assert_allclose(out["logits"], ref, rtol=0, atol=1e-13)
    for l in range(L):
        np.testing.assert_allclose(out["h"][l], hn[l, 0].numpy(), rtol=0, atol=1e-14)


# ----------------------------------------------------------------------------- P3 (trees)
def _tree_w(h=8, V=16, seed=0):
    return gen.tree_weights(h, V, seed, bf16=False)


def _caterpillar(n_right_leaves):
    """leaf0, leaf1, int(0,1), leaf3, int(2,3), ... post-order; root last."""
    left, right = [-1, -1, 0], [-1, -1, 1]
    for _ in range(n_right_leaves - 1):
        leaf = len(left)
        left.append(-1)
        right.append(-1)
        left.append(leaf - 1)
        right.append(leaf)
    return np.array(left), np.array(right)


def test_p3_caterpillar_reduces_to_lstm_cell():
    """Right leaves embed token 0 with E[0] = 0 and the leaf u-bias 0, so they output
    h = c = 0; every internal node is then LSTMCell(x = 0, h_L, c_L) with gates
    (i, f, g, o) <- (i, f_L, u, o) read from U[:, :h]; the leftmost leaf is
    LSTMCell(x, 0, 0) with (i, f, g, o) <- (i, -, u, o) read from W_leaf."""
    h = 8
    w = _tree_w(h)
    w.E[0] = 0
    w.b_leaf[2 * h:3 * h] = 0
    left, right = _caterpillar(5)
    toks = np.zeros(len(left), np.int64)
    toks[0] = 7
    root_h, root_c, _ = cells.tree_lstm(w, toks, left, right)

    leaf = torch.nn.LSTMCell(h, h, dtype=torch.float64)
    intern = torch.nn.LSTMCell(h, h, dtype=torch.float64)
    with torch.no_grad():
        Wl = torch.from_numpy(w.W_leaf.astype(np.float64))
        bl = torch.from_numpy(w.b_leaf.astype(np.float64))
        z = torch.zeros(h, h, dtype=torch.float64)
        leaf.weight_ih.copy_(torch.cat([Wl[0:h], z, Wl[2 * h:3 * h], Wl[h:2 * h]]))
        leaf.bias_ih.copy_(torch.cat([bl[0:h], torch.zeros(h, dtype=torch.float64),
                                      bl[2 * h:3 * h], bl[h:2 * h]]))
        leaf.weight_hh.zero_()
        leaf.bias_hh.zero_()
        U = torch.from_numpy(w.U.astype(np.float64))[:, :h]
        b = torch.from_numpy(w.b_int.astype(np.float64))
        intern.weight_hh.copy_(torch.cat([U[0:h], U[h:2 * h], U[4 * h:5 * h], U[3 * h:4 * h]]))
        intern.bias_hh.copy_(torch.cat([b[0:h], b[h:2 * h], b[4 * h:5 * h], b[3 * h:4 * h]]))
        intern.weight_ih.zero_()
        intern.bias_ih.zero_()
        x = torch.from_numpy(w.E[7].astype(np.float64))[None]
        zero = torch.zeros(1, h, dtype=torch.float64)
        th, tc = leaf(x, (zero, zero))
        for _ in range(5):
            th, tc = intern(zero, (th, tc))
    np.testing.assert_allclose(root_h, th[0].numpy(), rtol=0, atol=1e-14)
    np.testing.assert_allclose(root_c, tc[0].numpy(), rtol=0, atol=1e-14)


def _mirror(left, right):
    """Swap the children of every internal node and renumber into post-order."""
    n = len(left)
    nl, nr = [], []
    new_id = {}

    def visit(v):
        if left[v] < 0:
            nl.append(-1)
            nr.append(-1)
        else:
            a = visit(right[v])
            b = visit(left[v])
            nl.append(a)
            nr.append(b)
        new_id[v] = len(nl) - 1
        return new_id[v]

    visit(n - 1)
    perm = [None] * n
    for old, new in new_id.items():
        perm[new] = old
    return np.array(nl), np.array(nr), perm


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_p3_mirror_invariance(seed):
    """Mirroring the tree and swapping (U_L, f_L) <-> (U_R, f_R) gives the identical root."""
    h = 8
    w = _tree_w(h, seed=seed)
    rng = np.random.default_rng(seed)
    left, right = gen._random_bracketing(int(rng.integers(2, 9)), rng)
    toks = rng.integers(3, 16, size=len(left))
    rh, rc, _ = cells.tree_lstm(w, toks, left, right)
    ml, mr, perm = _mirror(left, right)
    mt = toks[perm]
    w2 = _tree_w(h, seed=seed)
    U = w.U.copy()
    w2.U = np.concatenate([U[:, h:], U[:, :h]], axis=1)
    w2.U[[*range(h, 2 * h), *range(2 * h, 3 * h)]] = w2.U[[*range(2 * h, 3 * h), *range(h, 2 * h)]]
    w2.b_int = w.b_int.copy()
    w2.b_int[h:3 * h] = np.concatenate([w.b_int[2 * h:3 * h], w.b_int[h:2 * h]])
    mh, mc, _ = cells.tree_lstm(w2, mt, ml, mr)
    np.testing.assert_allclose(mh, rh, rtol=0, atol=1e-12)
    np.testing.assert_allclose(mc, rc, rtol=0, atol=1e-12)


def test_p3_mirror_detects_asymmetric_child_use():
    """Sanity of the pin itself: a TreeLSTM that (wrongly) used c_L for both forget terms
    is not mirror-invariant, so the mirror test above would catch that mistake."""
    h = 8
    w = _tree_w(h, seed=5)
    rng = np.random.default_rng(5)
    hL, cL, hR, cR = (rng.standard_normal(h) for _ in range(4))

    def wrong(U, b, hl, cl, hr, cr):
        return cells.tree_internal(U, b, hl, cl, hr, cl)

    a = wrong(w.U, w.b_int, hL, cL, hR, cR)[1]
    U2 = np.concatenate([w.U[:, h:], w.U[:, :h]], axis=1)
    U2[[*range(h, 3 * h)]] = U2[[*range(2 * h, 3 * h), *range(h, 2 * h)]]
    b2 = w.b_int.copy()
    b2[h:3 * h] = np.concatenate([w.b_int[2 * h:3 * h], w.b_int[h:2 * h]])
    b = wrong(U2, b2, hR, cR, hL, cL)[1]
    assert np.max(np.abs(a - b)) > 1e-3


def test_p3_single_leaf_tree_is_leaf_cell():
    w = _tree_w(8)
    h, c, _ = cells.tree_lstm(w, [9], [-1], [-1])
    h2, c2 = cells.tree_leaf(w.W_leaf, w.b_leaf, w.E[9])
    np.testing.assert_array_equal(h, h2)
    np.testing.assert_array_equal(c, c2)


# ---------------------------------------------------------------- §8f N1: <eos> termination
def test_n1_seq2seq_eos_is_the_fixed_length_prefix():
    """L715: "Decoding terminates when either the <eos> symbol is generated or when the
    maximum decoding length is reached". With <eos> = v, the decode is the fixed-length decode
    (pinned by P2) cut right after the first step that emits v: same tokens, same logits, same
    final states as decoding exactly that many steps; a symbol never emitted changes nothing."""
    from oracle import cells
    enc = gen.lstm_stack_weights(32, 2, 16, seed=3, bf16=False, scale=4.0)
    dec = gen.lstm_stack_weights(32, 2, 16, seed=103, projection=True, bf16=False, scale=4.0)
    src = [3, 5, 7, 4]
    T = 12
    full = cells.seq2seq(enc, dec, src, T)
    y = full["tokens"]
    assert len(set(y)) >= 4  # several distinct symbols: several cut points
    for v in sorted(set(y)):
        e = y.index(v)
        cut = cells.seq2seq(enc, dec, src, T, eos_id=v)
        ref = cells.seq2seq(enc, dec, src, e + 1)
        assert cut["tokens"] == y[:e + 1] and cut["tokens"][-1] == v
        assert np.array_equal(cut["logits"], ref["logits"])
        for l in range(2):
            assert np.array_equal(cut["h"][l], ref["h"][l]) and np.array_equal(cut["c"][l], ref["c"][l])
    never = [v for v in range(16) if v not in y]
    if never:
        out = cells.seq2seq(enc, dec, src, T, eos_id=never[0])
        assert out["tokens"] == y and np.array_equal(out["h"][1], full["h"][1])
    # forced-token mode terminates on the forced (device) tokens
    forced = list(y)
    forced[1] = 13
    out = cells.seq2seq(enc, dec, src, T, forced_tokens=forced, eos_id=13)
    assert len(out["tokens"]) == 2
