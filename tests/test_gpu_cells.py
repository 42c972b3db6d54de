"""Kernel-level parity (-m gpu): ONE batched cell step through the C-ABI (bm_cell_step) over
arbitrary, non-contiguous pool slots, compared element by element with the fp64 oracle run on
exactly the values the device holds (bf16 weights/activations widened to fp64; fp32 c).

Sizes span several tiles and ragged tails: b across the 16-column MMA granularity and the
256-column CTA split, h = 64 (configs[0]) and h = 1024 (configs[1]-[4])."""
import numpy as np
import pytest

from oracle import cells
from paper_conf_eurosys_gaoywl18_b200 import bm
from gpu_helpers import TOL, bf16_vals, lstm_engine, tree_engine
from workloads import gen

pytestmark = pytest.mark.gpu

# result rows are fp32 straight from the epilogue: only fp32 accumulation/transcendental error
STEP_TOL = {bm.PREC_BF16: 2e-4, bm.PREC_FP32: 1e-5}


def _slots(rng, b, n_slots):
    return rng.choice(n_slots, size=b, replace=False).astype(np.int32)


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
@pytest.mark.parametrize("h,b", [(64, 1), (64, 17), (1024, 1), (1024, 15), (1024, 16), (1024, 17),
                                 (1024, 129), (1024, 256), (1024, 300), (1024, 512)])
def test_lstm_step_parity(prec, h, b):
    rng = np.random.default_rng(h * 1000 + b)
    V = 256
    e, cid, w = lstm_engine(h, 1, V, prec)
    slots = _slots(rng, b, 4096)
    par = rng.integers(0, 2, size=b)
    first = rng.random(b) < 0.2
    h0 = bf16_vals(rng.uniform(-1, 1, (b, h)), prec)
    c0 = rng.uniform(-2, 2, (b, h)).astype(np.float32)
    for p in (0, 1):
        m = par == p
        if m.any():
            e.pool_write(0, p, slots[m], h0[m], c0[m])
    toks = rng.integers(3, V, size=b)
    flags = (first * bm.ROW_FIRST) | bm.ROW_LAST | (par * bm.ROW_PARITY) | (np.arange(b) << 8)
    rows = np.stack([toks, np.zeros(b), slots, flags], 1).astype(np.int32)
    e.cell_step(cid, rows)
    rh, rc = e.result_rows(np.arange(b))
    ph = np.zeros((b, h), np.float32)
    for p in (0, 1):
        m = par == p
        if m.any():
            ph[m] = e.pool_read(0, 1 - p, slots[m])[0]
    pc = e.pool_read(0, 0, slots)[1]
    for i in range(b):
        hp = np.zeros(h) if first[i] else h0[i]
        cp = np.zeros(h) if first[i] else c0[i]
        eh, ec = cells.lstm_cell(w.W[0], w.b[0], w.E[toks[i]], hp, cp)
        assert np.max(np.abs(rh[i, 0] - eh)) <= STEP_TOL[prec], i
        assert np.max(np.abs(rc[i, 0] - ec)) <= STEP_TOL[prec], i
        assert np.max(np.abs(pc[i] - ec)) <= STEP_TOL[prec], i
        assert np.max(np.abs(ph[i] - eh)) <= TOL[prec], i   # pool h is stored in bf16


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
def test_lstm_stack_step_parity(prec):
    """One timestep of a 4-layer stack: layer l reads layer l-1's fresh h (A11)."""
    rng = np.random.default_rng(4)
    h, L, V, b = 1024, 4, 512, 40
    e, cid, w = lstm_engine(h, L, V, prec, max_slots=256, max_requests=256)
    slots = _slots(rng, b, 256)
    h0 = [bf16_vals(rng.uniform(-1, 1, (b, h)), prec) for _ in range(L)]
    c0 = [rng.uniform(-1, 1, (b, h)).astype(np.float32) for _ in range(L)]
    for l in range(L):
        e.pool_write(l, 1, slots, h0[l], c0[l])
    toks = rng.integers(3, V, size=b)
    flags = bm.ROW_LAST | bm.ROW_PARITY | (np.arange(b) << 8)
    e.cell_step(cid, np.stack([toks, np.zeros(b), slots, flags], 1))
    rh, rc = e.result_rows(np.arange(b))
    for i in range(b):
        x = w.E[toks[i]].astype(np.float64)
        for l in range(L):
            eh, ec = cells.lstm_cell(w.W[l], w.b[l], x, h0[l][i], c0[l][i])
            # every layer is one step on exactly the operands the device used (layer l > 0
            # consumes the stored bf16 h of layer l-1, read back below): single-step tolerance
            assert np.max(np.abs(rc[i, l] - ec)) <= STEP_TOL[prec], (i, l)
            assert np.max(np.abs(rh[i, l] - eh)) <= STEP_TOL[prec], (i, l)
            # the next layer consumes the device's stored (bf16) h, as the kernel does
            x = e.pool_read(l, 0, slots[i:i + 1])[0][0].astype(np.float64)


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
@pytest.mark.parametrize("b", [1, 33, 64, 200])
def test_tree_cells_parity(prec, b):
    rng = np.random.default_rng(b)
    h, V = 1024, 300
    e, (leaf, intern), w = tree_engine(h, V, prec, bmax=512, max_slots=2048, max_requests=2048)
    # leaves -> slots A ; internal nodes combine random pairs of them -> slots B
    A = _slots(rng, 2 * b, 1024)
    toks = rng.integers(3, V, size=2 * b)
    flags = bm.ROW_LAST | (np.arange(2 * b) << 8)
    e.cell_step(leaf, np.stack([toks, np.zeros(2 * b), A, flags], 1))
    lh, lc = e.result_rows(np.arange(2 * b))
    for i in range(2 * b):
        eh, ec = cells.tree_leaf(w.W_leaf, w.b_leaf, w.E[toks[i]])
        assert np.max(np.abs(lh[i, 0] - eh)) <= STEP_TOL[prec]
        assert np.max(np.abs(lc[i, 0] - ec)) <= STEP_TOL[prec]
    hA, cA = e.pool_read(0, 0, A)
    Bs = (1024 + _slots(rng, b, 1024)).astype(np.int32)
    L_, R_ = A[:b], A[b:]
    flags = bm.ROW_LAST | ((1000 + np.arange(b)) << 8)
    e.cell_step(intern, np.stack([L_, R_, Bs, flags], 1))
    ih, ic = e.result_rows(1000 + np.arange(b))
    for i in range(b):
        eh, ec = cells.tree_internal(w.U, w.b_int, hA[i], cA[i], hA[b + i], cA[b + i])
        assert np.max(np.abs(ih[i, 0] - eh)) <= STEP_TOL[prec]
        assert np.max(np.abs(ic[i, 0] - ec)) <= STEP_TOL[prec]


@pytest.mark.parametrize("prec", [bm.PREC_BF16, bm.PREC_FP32])
@pytest.mark.parametrize("b", [1, 37, 256])
def test_projection_argmax_parity(prec, b):
    """Decoder output projection + argmax (A10): h^L . W_out^T + b_out, argmax with the lowest
    index on ties, written to the device feed token tok[slot]. The device's choice must be a
    valid argmax of the fp64 logits within the tolerance (SURVEY §8c forced-token mode)."""
    rng = np.random.default_rng(b + 7)
    h, V = 1024, 32768
    e, cid, w = lstm_engine(h, 1, V, prec, proj=True, max_slots=1024, max_requests=1024,
                            record_logits=1, max_decode_len=4)
    slots = _slots(rng, b, 1024)
    h0 = bf16_vals(rng.uniform(-1, 1, (b, h)), prec)
    c0 = rng.uniform(-1, 1, (b, h)).astype(np.float32)
    e.pool_write(0, 0, slots, h0, c0)
    toks = rng.integers(3, V, size=b)
    flags = bm.ROW_PARITY | (np.arange(b) << 8)   # reads parity 1, writes parity 0
    e.pool_write(0, 1, slots, h0, c0)
    e.cell_step(cid, np.stack([toks, np.full(b, 2), slots, flags], 1))
    hn = e.pool_read(0, 0, slots)[0]            # the layer's fresh h (device values)
    y = e.tokens(slots)
    tol = TOL[prec]
    for i in range(b):
        lg = w.W_out.astype(np.float64) @ hn[i].astype(np.float64) + w.b_out
        assert lg[y[i]] >= lg.max() - 2 * tol, (i, lg[y[i]], lg.max())


@pytest.mark.parametrize("b", [16, 100, 128])
def test_batch_invariance_bitwise(b):
    """P10: a row's bf16 result is bitwise identical whatever else shares its task (single-CTA
    regime, tasks of <= 128 rows; the CTA-pair regime is tested below)."""
    rng = np.random.default_rng(11)
    h, V = 1024, 256
    e, cid, w = lstm_engine(h, 1, V, bm.PREC_BF16)
    slots = _slots(rng, b, 4096)
    h0 = bf16_vals(rng.uniform(-1, 1, (b, h)), bm.PREC_BF16)
    c0 = rng.uniform(-1, 1, (b, h)).astype(np.float32)
    toks = rng.integers(3, V, size=b)
    e.pool_write(0, 0, slots, h0, c0)
    flags = bm.ROW_LAST | (np.arange(b) << 8)
    e.cell_step(cid, np.stack([toks, np.zeros(b), slots, flags], 1))
    full_h, full_c = e.result_rows(np.arange(b))
    e.pool_write(0, 0, slots[:1], h0[:1], c0[:1])
    e.cell_step(cid, np.array([[toks[0], 0, slots[0], bm.ROW_LAST | (4000 << 8)]]))
    one_h, one_c = e.result_rows([4000])
    assert np.array_equal(one_h[0], full_h[0])
    assert np.array_equal(one_c[0], full_c[0])


@pytest.mark.parametrize("b_small,b_big", [(260, 512), (300, 384), (129, 256), (200, 512)])
def test_batch_invariance_pair_regime(b_small, b_big):
    """P10 for the CTA-pair kernel (tasks of 129..512 rows, tcgen05.mma.cta_group::2, S = 2): a
    row's result is bitwise identical in a task of b_small and of b_big rows (the column block
    and pair half it lands in differ; its K-order and split-K order do not)."""
    rng = np.random.default_rng(12)
    h, V = 1024, 256
    e, cid, w = lstm_engine(h, 1, V, bm.PREC_BF16)
    slots = _slots(rng, b_big, 4096)
    h0 = bf16_vals(rng.uniform(-1, 1, (b_big, h)), bm.PREC_BF16)
    c0 = rng.uniform(-1, 1, (b_big, h)).astype(np.float32)
    toks = rng.integers(3, V, size=b_big)
    flags = bm.ROW_LAST | (np.arange(b_big) << 8)
    rows = np.stack([toks, np.zeros(b_big), slots, flags], 1)
    e.pool_write(0, 0, slots, h0, c0)
    e.cell_step(cid, rows)
    big_h, big_c = e.result_rows(np.arange(b_big))
    # the same first rows again, now the LAST b_small rows of a smaller task (other columns)
    sel = np.concatenate([np.arange(b_small - 40, b_small), np.arange(0, b_small - 40)])
    e.pool_write(0, 0, slots, h0, c0)
    e.cell_step(cid, rows[sel])
    small_h, small_c = e.result_rows(np.arange(b_big)[sel])
    assert np.array_equal(small_h, big_h[sel])
    assert np.array_equal(small_c, big_c[sel])
    # and within tolerance of the oracle
    for i in (0, b_small - 1):
        hs, cs = cells.lstm_cell(w.W[0].astype(np.float64), w.b[0].astype(np.float64),
                                 w.E[toks[i]].astype(np.float64), h0[i].astype(np.float64),
                                 c0[i].astype(np.float64))
        assert np.max(np.abs(big_h[i] - hs)) <= STEP_TOL[bm.PREC_BF16]
        assert np.max(np.abs(big_c[i] - cs)) <= STEP_TOL[bm.PREC_BF16]


@pytest.mark.parametrize("b_small,b_big", [(1, 64), (37, 256)])
def test_leaf_batch_invariance(b_small, b_big):
    """P10 for the TreeLSTM leaf cell (256-wide K slices, S = 4, tasks of <= 256 rows): a leaf's
    result is bitwise identical in a task of b_small and of b_big rows, and within tolerance of
    the oracle."""
    rng = np.random.default_rng(13)
    h, V = 1024, 300
    e, (leaf, intern), w = tree_engine(h, V, bm.PREC_BF16, bmax=512, max_slots=2048, max_requests=2048)
    slots = _slots(rng, b_big, 2048)
    toks = rng.integers(3, V, size=b_big)
    flags = bm.ROW_LAST | (np.arange(b_big) << 8)
    rows = np.stack([toks, np.zeros(b_big), slots, flags], 1)
    e.cell_step(leaf, rows)
    big_h, big_c = e.result_rows(np.arange(b_big))
    sel = np.arange(b_small)[::-1]
    e.cell_step(leaf, rows[sel])
    small_h, small_c = e.result_rows(np.arange(b_big)[sel])
    assert np.array_equal(small_h, big_h[sel])
    assert np.array_equal(small_c, big_c[sel])
    for i in (0, b_small - 1, b_big - 1):
        eh, ec = cells.tree_leaf(w.W_leaf, w.b_leaf, w.E[toks[i]])
        assert np.max(np.abs(big_h[i, 0] - eh)) <= STEP_TOL[bm.PREC_BF16]
        assert np.max(np.abs(big_c[i, 0] - ec)) <= STEP_TOL[bm.PREC_BF16]


def test_lstm_step_every_batch_size():
    """Every task size the scheduler can form, b = 1..512 (bmax), one LSTM step at h = 1024
    through whichever kernel and plan the launcher picks for that b (single-CTA tcgen05 with
    its ring plans, CTA pair above 128 rows, one or two column blocks, ragged tails): result
    rows (fp32) against the oracle at single-step tolerance, pool h (bf16) at north_star's."""
    from oracle import batched
    rng = np.random.default_rng(77)
    h, V = 1024, 512
    e, cid, w = lstm_engine(h, 1, V, bm.PREC_BF16, max_slots=2048, max_requests=1024)
    worst = {}
    for b in range(1, 513):
        slots = _slots(rng, b, 2048)
        first = rng.random(b) < 0.1
        h0 = bf16_vals(rng.uniform(-1, 1, (b, h)), bm.PREC_BF16)
        c0 = rng.uniform(-2, 2, (b, h)).astype(np.float32)
        e.pool_write(0, 0, slots, h0, c0)
        toks = rng.integers(3, V, size=b)
        flags = (first * bm.ROW_FIRST) | bm.ROW_LAST | (np.arange(b) << 8)
        e.cell_step(cid, np.stack([toks, np.zeros(b), slots, flags], 1).astype(np.int32))
        rh, rc = e.result_rows(np.arange(b))
        ph = e.pool_read(0, 1, slots)[0]
        hp = np.where(first[:, None], 0.0, h0)
        cp = np.where(first[:, None], 0.0, c0)
        eh, ec = batched.lstm_step_rows(w.W[0], w.b[0], w.E[toks], hp, cp)
        err = max(np.max(np.abs(rh[:, 0] - eh)), np.max(np.abs(rc[:, 0] - ec)))
        worst[b] = (err, np.max(np.abs(ph - eh)))
    bad = {b: v for b, v in worst.items() if v[0] > STEP_TOL[bm.PREC_BF16] or v[1] > TOL[bm.PREC_BF16]}
    assert not bad, sorted(bad.items())[:10]
