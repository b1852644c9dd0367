"""Multi-GPU bootstrap: one process per GPU.

The path's only exchange step -- a7, the MIN all-reduce of the ranks' smallest
feasible candidate indices (and, for a batch, the all-gather of the winners'
allocations) -- runs inside libmadpipe over the ctx's own NCCL communicator
(madpipe_ctx_create with rank, world and an NCCL id).  So an N-GPU solve is one
C call per rank: ``context(...).solve_dev(...)``.  This module only does the
process bootstrap: rank 0 creates the 128-byte NCCL id (madpipe_get_unique_id)
and the launcher's process group (torch.distributed, any backend) carries it to
the other ranks.  Nothing here touches the DP's data.
"""
from __future__ import annotations

import torch.distributed as dist

from . import Context, get_unique_id


def share_id(group=None) -> bytes:
    """Rank 0's NCCL id, broadcast over the torch process group (bootstrap only)."""
    obj = [get_unique_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def context(device: int, stream=None, group=None, mem_budget: int = 0) -> Context:
    """A Context that is rank ``dist.get_rank(group)`` of ``dist.get_world_size(group)``
    with a communicator over all of them (also at world 1)."""
    nid = share_id(group)
    return Context(device, stream=stream, mem_budget=mem_budget, rank=dist.get_rank(group),
                   world=dist.get_world_size(group), nccl_id=nid)
