"""The N>1 controller (paper_conf_ipps_beaumontes22_b200/distributed.py) on CPU process
groups (gloo, world size 2 and 3).  The two library calls are replaced by oracle-backed
doubles; the sharding rule is the library's own (madpipe_shard, host-only) and the
exchange is the real all-reduce(MIN).  Every rank must obtain the world-1 answer."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as tmp

import chaingen
import oracle
import paper_conf_ipps_beaumontes22_b200 as mp
from paper_conf_ipps_beaumontes22_b200.distributed import INT32_MAX, solve_distributed


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _case(seed):
    rng = np.random.default_rng(seed)
    ch = chaingen.tiny(rng, 9)
    M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * (0.12 + 0.05 * seed))
    return ch, 3, M, 25.0, 4, 8, 20


def _worker(rank, world, port, seed, early_exit, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ch, P, M, beta, n_m, n_v, n_c = _case(seed)
    tau = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, j_lo=0, j_hi=1)["tau"]
    evaluated = []

    def sweep_fn(r, w, jl):
        best = INT32_MAX
        for j in mp.shard(n_c, r, w):
            A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, 0, tau[j], with_arg=False)
            evaluated.append(j)
            if A[-1, P - 1, 0, 0] <= tau[j]:
                best = min(best, j)
                if early_exit:
                    break
        jl.fill_(best)
        return len(evaluated)

    def resolve_fn(jl):
        j = int(jl.item())
        if j == INT32_MAX:
            return dict(rc=oracle.INFEASIBLE)
        r = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, j_lo=j, j_hi=j + 1)
        return dict(rc=r["rc"], cand_index=r["cand_index"], stages=r["stages"],
                    period=r["period"], special_load=r["special_load"])

    res, cu = solve_distributed(ch, P, M, beta, n_m, n_v, n_c, early_exit=early_exit,
                                device=torch.device("cpu"), sweep_fn=sweep_fn, resolve_fn=resolve_fn)
    out[rank] = (res, sorted(evaluated))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,early_exit,seed", [(2, False, 1), (2, True, 2), (3, False, 3),
                                                   (3, True, 4)])
def test_controller_matches_world1(world, early_exit, seed):
    ch, P, M, beta, n_m, n_v, n_c = _case(seed)
    ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c)
    with tmp.Manager() as mgr:
        out = mgr.dict()
        tmp.spawn(_worker, args=(world, _free_port(), seed, early_exit, out), nprocs=world, join=True)
        results = dict(out)
    assert len(results) == world
    evaluated = []
    for r in range(world):
        res, ev = results[r]
        evaluated += ev
        assert res["rc"] == ref["rc"]
        if ref["rc"] == 0:
            assert res["cand_index"] == ref["cand_index"]
            assert res["stages"] == ref["stages"]
            assert res["period"] == ref["period"] and res["special_load"] == ref["special_load"]
    if not early_exit:
        assert sorted(evaluated) == list(range(n_c))     # every candidate exactly once
    else:
        assert len(set(evaluated)) == len(evaluated)
