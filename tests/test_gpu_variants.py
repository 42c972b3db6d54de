"""The CTA-pair LSTM kernel's two weight paths give bit-identical results.

By default each stage's weight K blocks move by one bulk copy of the TMA warp (from kernel entry);
BM_PAIR_WTMA=0 moves them by the producers' cp.async next to the activation gather. The bytes
land in the same stage layout and the MMAs, the split-K order and the gate arithmetic are the
same, so every result row must match bit for bit at every pair-kernel batch size (b = 129..512,
ragged column blocks; tools/pair_cmp.py). The default path itself is checked against the oracle
by test_gpu_cells.py. Each variant runs in its own process (the launcher reads the variable once)."""
import os
import subprocess
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(tmp_path, name, env_extra):
    out = str(tmp_path / f"{name}.npz")
    env = dict(os.environ)
    env.pop("BM_PAIR_WTMA", None)
    env.update(env_extra)
    subprocess.run([sys.executable, os.path.join(ROOT, "tools", "pair_cmp.py"), out], env=env, check=True,
                   timeout=600)
    return np.load(out)


@pytest.mark.gpu
def test_pair_weight_paths_bitwise(tmp_path):
    ref = _run(tmp_path, "cp_async", {"BM_PAIR_WTMA": "0"})
    new = _run(tmp_path, "bulk", {})
    assert set(ref.files) == set(new.files) and len(ref.files) == 16
    for k in ref.files:
        assert np.array_equal(ref[k], new[k]), k
