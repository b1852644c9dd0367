"""Multi-GPU controller: one process per GPU.

Candidate periods are independent units, sharded interleaved (rank r owns
j = r, r+W, ...; the cost of a candidate grows with its period, so interleaving
balances the ranks).  Each rank sweeps its shard (madpipe_sweep), the ranks
min-reduce their smallest feasible candidate index with ONE all-reduce (the
path's only exchange step, a7: 4 bytes over NVLink with NCCL), and every rank
re-solves the winner and traces it back (madpipe_resolve) -- deterministic,
so no broadcast of the allocation is needed.

The same function runs on CPU process groups (gloo) in the tests, with the two
library calls replaced by test doubles (``sweep_fn`` / ``resolve_fn``).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

INT32_MAX = 2 ** 31 - 1


def solve_distributed(chain, P, M, beta, n_mem, n_delay, n_periods, v_range=0, early_exit=False,
                      ctx=None, group=None, device=None, sweep_fn=None, resolve_fn=None):
    """Returns (result dict, this rank's cell-update count)."""
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    if device is None:
        device = torch.device("cuda", torch.cuda.current_device())
    jl = torch.full((1,), INT32_MAX, dtype=torch.int32, device=device)
    if sweep_fn is None:
        cu = ctx.sweep(chain, P, M, beta, n_mem, n_delay, n_periods, rank, world, jl.data_ptr(),
                       v_range=v_range, early_exit=early_exit)
    else:
        cu = sweep_fn(rank, world, jl)
    dist.all_reduce(jl, op=dist.ReduceOp.MIN, group=group)        # a7
    if jl.is_cuda:
        torch.cuda.current_stream(jl.device).synchronize()
    if resolve_fn is None:
        res = ctx.resolve(chain, P, M, beta, n_mem, n_delay, n_periods, jl.data_ptr(),
                          v_range=v_range)
    else:
        res = resolve_fn(jl)
    return res, cu
