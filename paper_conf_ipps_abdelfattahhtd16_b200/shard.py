"""Multi-GPU sharding of a vbatched problem.

The matrices of a batch are independent, so the batch shards with no
data-path collective: each rank factors the matrices it owns. Ownership is a flop-balanced
longest-processing-time partition on n^3/3 computed by the library's native host helper
``vbatched_partition_lpt`` (identical on every rank, so no communication is needed to
agree on it). torch.distributed is used only for the barrier, the per-rank timings (max
over ranks) and the gather of (global index, info) pairs — NCCL on the GPU box, gloo in the
CPU tests.
"""
from __future__ import annotations

import numpy as np

from . import vbatched_partition_lpt


def lpt_owner(n_all, world: int) -> np.ndarray:
    """owner[i] in [0, world) for every matrix (native LPT, deterministic)."""
    n_all = np.ascontiguousarray(n_all, dtype=np.int32)
    if world == 1:
        return np.zeros(len(n_all), dtype=np.int32)
    return vbatched_partition_lpt(n_all, world)


def shard_indices(n_all, world: int, rank: int) -> np.ndarray:
    """Global indices owned by `rank`, in increasing order."""
    owner = lpt_owner(n_all, world)
    return np.nonzero(owner == rank)[0].astype(np.int32)


def shard_loads(n_all, world: int) -> np.ndarray:
    """Per-rank sum of n^3/3 under the LPT partition."""
    owner = lpt_owner(n_all, world)
    n = np.asarray(n_all, dtype=np.float64)
    return np.bincount(owner, weights=n ** 3 / 3.0, minlength=world)


def max_over_ranks(value: float, device=None) -> float:
    """Max of a per-rank scalar (e.g. the device-timed step time) over all ranks."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(value: float, device=None) -> float:
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def gather_info(batch: int, local_idx, local_info, device=None) -> np.ndarray:
    """Assemble the global info[] from every rank's (global index, info) pairs (all ranks get
    the full array). Ranks own disjoint index sets; every index must be owned once."""
    import torch
    import torch.distributed as dist
    local_idx = np.asarray(local_idx, dtype=np.int32)
    local_info = np.asarray(local_info, dtype=np.int32)
    out = np.full(batch, np.iinfo(np.int32).min, dtype=np.int32)
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        out[local_idx] = local_info
        return out
    world = dist.get_world_size()
    cnt = torch.tensor([len(local_idx)], dtype=torch.int64, device=device)
    cnts = [torch.zeros_like(cnt) for _ in range(world)]
    dist.all_gather(cnts, cnt)
    m = int(max(int(c.item()) for c in cnts))
    pairs = np.full((max(m, 1), 2), -1, dtype=np.int32)
    pairs[: len(local_idx), 0] = local_idx
    pairs[: len(local_idx), 1] = local_info
    t = torch.from_numpy(pairs).to(device) if device is not None else torch.from_numpy(pairs)
    allp = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(allp, t)
    for r, p in enumerate(allp):
        p = p.cpu().numpy()[: int(cnts[r].item())]
        out[p[:, 0]] = p[:, 1]
    return out
