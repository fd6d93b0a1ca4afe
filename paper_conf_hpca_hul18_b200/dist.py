"""Multi-GPU plumbing for the SFC path.

One process per GPU (torch.distributed).  Flows are partitioned by RSS
("Receive Side Steering"): shard = RETA[Toeplitz(MS key, tuple) & 127],
RETA[j] = j mod N -- computed on the GPU by nfc_rss_shard.  There is no
data-path collective: each rank runs its own chain on its own shard.  The only
collectives are one all-reduce (sum) of the u64 counter vector and a max of
the per-rank device times.  This module is host logic only (no packet compute).
"""
from __future__ import annotations

import os
from typing import Tuple

import numpy as np


def env_ranks() -> Tuple[int, int, int]:
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def reta(n_shards: int, size: int = 128) -> np.ndarray:
    """RSS redirection table: entry j -> shard j mod n_shards."""
    if not 1 <= n_shards <= size:
        raise ValueError("n_shards must be 1..128")
    return np.arange(size, dtype=np.int64) % n_shards


def shard_of_hash(h: np.ndarray, n_shards: int) -> np.ndarray:
    return reta(n_shards)[np.asarray(h, dtype=np.int64) & 127]


def shard_indices(shard_ids: np.ndarray, rank: int) -> np.ndarray:
    """Global indices of this rank's packets, in global order (stable)."""
    return np.nonzero(np.asarray(shard_ids) == rank)[0]


def allreduce_stats(stats: np.ndarray, device=None, group=None) -> np.ndarray:
    """Sum the u64 counter vector over ranks (one collective)."""
    import torch
    import torch.distributed as dist
    t = torch.from_numpy(np.ascontiguousarray(stats, dtype=np.uint64).view(np.int64).copy())
    if device is not None:
        t = t.to(device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return t.cpu().numpy().view(np.uint64)


def max_over_ranks(x: float, device=None, group=None) -> float:
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def library_comm(device: int):
    """The library's own NCCL communicator for this rank (nfc_comm_init): rank 0 makes
    the id (nfc_comm_unique_id) and torch.distributed broadcasts it.  Attach it to a
    chain with Chain.attach_comm; Chain.stats(allreduce=True) then sums the counters
    of every rank with one ncclAllReduce inside the library."""
    import torch.distributed as dist
    from paper_conf_hpca_hul18_b200 import nfc
    rank, world = dist.get_rank(), dist.get_world_size()
    box = [nfc.comm_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(box, src=0)
    return nfc.Comm(device, world, rank, box[0])


def merge_by_index(parts, n_total: int, dtype) -> np.ndarray:
    """parts = [(global_indices, records)] from every rank -> records in global order."""
    out = np.zeros(n_total, dtype=dtype)
    seen = np.zeros(n_total, dtype=bool)
    for idx, rec in parts:
        if np.any(seen[idx]):
            raise ValueError("a packet was processed by two ranks")
        out[idx] = rec
        seen[idx] = True
    if not seen.all():
        raise ValueError("a packet was processed by no rank")
    return out
