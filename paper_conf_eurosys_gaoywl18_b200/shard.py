"""Request sharding over GPUs — host-side plumbing only.

The cellular-batching path shards by request: requests are independent and no cell step ever
needs another request's state, so each rank runs its own engine (Algorithm 1 with one worker,
its own slot pool and weight replica) over its own Poisson stream. The only collectives are
off the per-step path:
  * one broadcast of the weight arrays from rank 0 at load time (NCCL over NVLink on GPUs,
    gloo in the CPU tests),
  * max-over-ranks reductions of timings and a gather of latency samples at the end.
The paper's own multi-GPU design (one manager, many workers, subgraph pinning and cross-GPU
state migration, L317-L381) is SURVEY §8f row N2 (bm_config.workers).
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

import numpy as np


def rank_seed(base: int, rank: int) -> int:
    """Independent, reproducible trace seed per rank (weak scaling: every rank offers the same
    per-GPU load from its own stream)."""
    return base + 7919 * rank


def broadcast_arrays(arrays: Sequence[Tuple[str, np.ndarray]], dist, device=None) -> None:
    """Overwrite every array on every rank with rank 0's values (in place). `device`: torch
    device for the collective's buffers (cuda for NCCL, None = cpu for gloo)."""
    import torch
    rank = dist.get_rank()
    for _, arr in arrays:
        if rank == 0:
            t = torch.from_numpy(np.ascontiguousarray(arr))
            t = t.to(device) if device is not None else t.clone()
        else:
            t = torch.empty(arr.shape, dtype=torch.from_numpy(arr[:0]).dtype,
                            device=device if device is not None else "cpu")
        dist.broadcast(t, src=0)
        if rank != 0:
            arr[...] = t.cpu().numpy()


def broadcast_tensors(arrays: Sequence[Tuple[str, np.ndarray]], dist, device=None) -> dict:
    """Rank 0's arrays on every rank as tensors on `device` (NCCL over NVLink: the weights land
    in device memory and bm_load_cell adopts them in place, include/bm.h bm_weights). With
    device None (gloo on CPU) the numpy arrays are also overwritten in place."""
    import torch
    rank = dist.get_rank()
    out = {}
    for name, arr in arrays:
        if rank == 0:
            t = torch.from_numpy(np.ascontiguousarray(arr))
            t = t.to(device) if device is not None else t.clone()
        else:
            t = torch.empty(arr.shape, dtype=torch.from_numpy(arr[:0]).dtype,
                            device=device if device is not None else "cpu")
        dist.broadcast(t, src=0)
        if device is None and rank != 0:
            arr[...] = t.numpy()
        out[name] = t
    return out


def reduce_max(x: float, dist=None, device=None) -> float:
    if dist is None:
        return x
    import torch
    t = torch.tensor([x], dtype=torch.float64, device=device if device is not None else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def reduce_sum(x: float, dist=None, device=None) -> float:
    if dist is None:
        return x
    import torch
    t = torch.tensor([x], dtype=torch.float64, device=device if device is not None else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def gather_samples(a: np.ndarray, dist=None, device=None) -> np.ndarray:
    """Concatenate every rank's latency samples (variable length) on every rank."""
    if dist is None:
        return np.asarray(a, np.float64)
    import torch
    world = dist.get_world_size()
    dev = device if device is not None else "cpu"
    n = torch.tensor([len(a)], dtype=torch.int64, device=dev)
    ns = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(ns, n)
    m = int(max(int(x.item()) for x in ns))
    buf = torch.zeros(m, dtype=torch.float64, device=dev)
    buf[:len(a)] = torch.from_numpy(np.asarray(a, np.float64)).to(dev)
    bufs = [torch.zeros_like(buf) for _ in range(world)]
    dist.all_gather(bufs, buf)
    return np.concatenate([b[:int(k.item())].cpu().numpy() for b, k in zip(bufs, ns)])


def percentiles(lat: np.ndarray, qs=(50, 90, 99)) -> List[float]:
    return [float(np.percentile(lat, q)) if len(lat) else float("nan") for q in qs]
