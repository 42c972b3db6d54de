"""The C-ABI library loads and exports every entry point include/bm.h declares; without an
sm_100 device, every device-backed engine fails loudly (BM_E_NODEV) — there is no CPU fallback."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "bm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bm_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_paper_boundary():
    names = _declared()
    for n in ("bm_load_cell", "bm_submit", "bm_schedule_step", "bm_poll"):
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_eurosys_gaoywl18_b200 import bm
    lib = ctypes.CDLL(bm.LIB_PATH)
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing
    assert lib.bm_abi_version() == 1


def test_binding_covers_every_declared_symbol():
    from paper_conf_eurosys_gaoywl18_b200 import bm
    assert sorted(bm._SIGS) == _declared()


def test_no_device_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_eurosys_gaoywl18_b200 import bm
    with pytest.raises(bm.BMError) as ei:
        bm.Engine(clock=bm.CLOCK_WALL, hidden=64, max_slots=16, max_requests=16)
    assert ei.value.status == bm.E_NODEV


def test_invalid_arguments_rejected():
    from paper_conf_eurosys_gaoywl18_b200 import bm
    with pytest.raises(bm.BMError):
        bm.Engine(clock=bm.CLOCK_DRY, hidden=100)  # h must be a multiple of 64
    import numpy as np
    e = bm.Engine(clock=bm.CLOCK_DRY, hidden=64, max_slots=16, max_requests=4)
    W = [np.zeros((256, 128), np.float32)]
    b = [np.zeros(256, np.float32)]
    E = np.zeros((10, 64), np.float32)
    cid = e.load_cell(bm.CELL_LSTM, 1, 10, 4, 0, W, b, E)
    with pytest.raises(bm.BMError):
        e.submit(bm.REQ_CHAIN, cid, 0, [3, 99])          # token >= vocab
    with pytest.raises(bm.BMError):
        e.submit(bm.REQ_TREE, cid, cid, [3, 3, 3], left=[-1, -1, 0], right=[-1, -1, 1])
    with pytest.raises(bm.BMError):
        e.load_cell(bm.CELL_LSTM, 2, 10, 4, 0, W * 2, b * 2, E)   # layers > pool_layers
    for _ in range(4):
        e.submit(bm.REQ_CHAIN, cid, 0, [3])
    with pytest.raises(bm.BMError) as ei:
        e.submit(bm.REQ_CHAIN, cid, 0, [3])              # table full: back-pressure
    assert ei.value.status == bm.E_FULL
    with pytest.raises(bm.BMError) as ei:
        e.load_cell(bm.CELL_LSTM, 1, 10, 4, 0, W, b, E)  # cells must precede submits
    assert ei.value.status == bm.E_STATE


def test_malformed_trees_rejected():
    import numpy as np
    from paper_conf_eurosys_gaoywl18_b200 import bm
    e = bm.Engine(clock=bm.CLOCK_DRY, hidden=64, max_slots=64, max_requests=16)
    leaf = e.load_cell(bm.CELL_TREE_LEAF, 1, 10, 8, 0, [np.zeros((192, 64), np.float32)],
                       [np.zeros(192, np.float32)], np.zeros((10, 64), np.float32))
    intern = e.load_cell(bm.CELL_TREE_INTERNAL, 1, 10, 8, 1, [np.zeros((320, 128), np.float32)],
                         [np.zeros(320, np.float32)])
    bad = [([-1, -1, 1], [-1, -1, 0]),        # root children not post-order distinct? (1, 0) ok?
           ([-1, 0, -1], [-1, -1, -1]),       # one-child node
           ([-1, -1, 2], [-1, -1, 1]),        # self reference
           ([-1, -1, -1], [-1, -1, -1])]      # forest (no single root)
    for left, right in bad[1:]:
        with pytest.raises(bm.BMError):
            e.submit(bm.REQ_TREE, leaf, intern, [3, 3, 3], left=left, right=right)
    e.submit(bm.REQ_TREE, leaf, intern, [3, 4, 0], left=[-1, -1, 1], right=[-1, -1, 0])


def test_poll_array_layout_matches_bm_completion():
    """bm.Engine.poll_array views bm_completion records as a numpy structured array: the dtype
    must mirror the C struct (field order, offsets, size)."""
    import ctypes as C
    from paper_conf_eurosys_gaoywl18_b200 import bm
    dt = bm.Engine._COMP_DT
    assert dt.itemsize == C.sizeof(bm.Completion)
    for name, _ in bm.Completion._fields_:
        assert dt.fields[name][1] == getattr(bm.Completion, name).offset
