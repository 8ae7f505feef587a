"""Row sharding of the sample over one process per GPU.

The sample is split into contiguous row blocks, one per rank; query boxes,
h and parameters are replicated; per-box partial sums (S_0, S_j) are combined
inside libkde with an all-gather + fixed-order sum, so every rank gets
identical, deterministic results.  The all-gather runs over peer device memory
(libkde's own kernels, default) or NCCL.  torch.distributed is plumbing only: it
bootstraps the process group and exchanges the IPC handles / ncclUniqueId.
"""
from __future__ import annotations

from . import KDEModel, kde_get_unique_id


def shard_range(n_global: int, rank: int, world: int):
    """Contiguous balanced split: rank r owns rows [off, off + n) with the
    first (n_global % world) ranks holding one extra row."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    base, extra = divmod(n_global, world)
    off = rank * base + min(rank, extra)
    return off, base + (1 if rank < extra else 0)


def exchange_unique_id(get_id=kde_get_unique_id) -> bytes:
    """Rank 0 creates the ncclUniqueId; every rank receives it through the
    torch.distributed default group (works for the gloo and nccl backends)."""
    import torch.distributed as dist
    obj = [get_id() if dist.get_rank() == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    return obj[0]


def all_gather_bytes(b: bytes):
    """Every rank's bytes, in rank order, through the torch.distributed default group."""
    import torch.distributed as dist
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, b)
    return out


def create_sharded(local_rows, row_offset: int, n_global: int, h=None, transport: str = "peer") -> KDEModel:
    """Collective: build this rank's shard of a model over n_global rows.
    transport "peer": the library's own exchange over peer device memory (IPC
    handles all-gathered here); "nccl": ncclAllGather (ncclUniqueId broadcast here)."""
    import torch.distributed as dist
    rank, world = dist.get_rank(), dist.get_world_size()
    if transport == "peer":
        return KDEModel.create_sharded_peer(local_rows, row_offset, n_global, h, rank, world, all_gather_bytes)
    if transport != "nccl":
        raise ValueError(f"unknown transport {transport!r}")
    nid = exchange_unique_id() if world > 1 else None
    return KDEModel.create_sharded(local_rows, row_offset, n_global, h, nid, rank, world)
