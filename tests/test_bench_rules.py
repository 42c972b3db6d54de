"""bench.py's sustained-load rule on synthetic completion records: a system that
keeps up completes at the offered rate with a flat backlog; an overloaded one completes at its
capacity and its backlog trend grows with the window. Host logic only (no engine, no GPU)."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def _fifo(lam, mu, n, seed):
    """Poisson arrivals at rate lam, one FIFO server with exponential service at rate mu
    (M/M/1): the completion times of the n requests."""
    rng = np.random.default_rng(seed)
    ta = np.cumsum(rng.exponential(1.0 / lam, n))
    svc = rng.exponential(1.0 / mu, n)
    td = np.empty(n)
    t = 0.0
    for i in range(n):
        t = max(t, ta[i]) + svc[i]
        td[i] = t
    return {"t_arrival": ta, "t_done": td}


def _sustained(comp, lam):
    rate, _, _, mean, growth = bench.steady_rate(comp)
    return rate >= bench.SUSTAINED * lam and growth <= bench.BACKLOG_GROWTH * mean + 64, rate, growth


def test_stable_system_is_sustained():
    lam = 1000.0
    ok, rate, growth = _sustained(_fifo(lam, 1500.0, 200_000, 1), lam)
    assert ok, (rate, growth)
    assert abs(rate / lam - 1) < 0.02


def test_overloaded_system_is_not_sustained():
    lam, mu = 1000.0, 900.0
    ok, rate, growth = _sustained(_fifo(lam, mu, 200_000, 2), lam)
    assert not ok
    assert abs(rate / mu - 1) < 0.02          # completions at capacity, not at the offered rate
    assert growth > 0.05 * (lam - mu) * 180   # the queue grows ~ (lam - mu) x window


def test_drain_is_not_charged():
    # every request takes the same long latency: n / (first arrival .. last completion) is
    # below the offered rate, the steady-state rate is not, and the backlog is flat
    lam = 1000.0
    rng = np.random.default_rng(3)
    ta = np.cumsum(rng.exponential(1.0 / lam, 100_000))
    comp = {"t_arrival": ta, "t_done": ta + 2.0}
    ok, rate, growth = _sustained(comp, lam)
    assert ok and abs(rate / lam - 1) < 0.02
    assert 100_000 / (comp["t_done"].max() - ta.min()) < 0.99 * lam
