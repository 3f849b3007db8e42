"""Host-side multi-GPU plumbing (one process per GPU, torch.distributed).

* mode 0, replicate / source sharding: every rank builds the graph and answers a
  contiguous block of the sources -- `shard_sources`; no data-path collective.
* mode 1, vertex range: one query batch partitioned by vertex range; the C-ABI
  exchanges states with ncclAllReduce(min) -- `make_comm` creates the NCCL
  communicator from a unique id broadcast over the process group.
`max_over_ranks` is the timing reduction the bench uses.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_sources(sources, rank: int, world: int):
    """Contiguous block of `sources` for `rank` (blocks differ by at most one)."""
    k = len(sources)
    lo = (k * rank) // world
    hi = (k * (rank + 1)) // world
    return list(sources[lo:hi])


def broadcast_bytes(data: bytes | None, nbytes: int, src: int = 0, device=None) -> bytes:
    """Broadcast `nbytes` raw bytes from rank `src` over the default process group."""
    t = torch.zeros(nbytes, dtype=torch.uint8, device=device)
    if dist.get_rank() == src:
        t.copy_(torch.frombuffer(bytearray(data), dtype=torch.uint8).to(t.device))
    dist.broadcast(t, src)
    return bytes(t.cpu().tolist())


def max_over_ranks(value: float, device=None) -> float:
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def make_comm(rank: int, world: int, device: int, bcast_device=None):
    """NCCL communicator of the C-ABI for (rank, world) on `device`."""
    from . import tempgraph as tg
    uid = tg.tg_nccl_unique_id() if rank == 0 else None
    if world > 1:
        uid = broadcast_bytes(uid, 128, 0, device=bcast_device)
    return tg.tg_comm_create(uid, rank, world, device)
