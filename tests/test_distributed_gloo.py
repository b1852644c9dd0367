"""The N>1 protocol on CPU process groups (gloo, world size 2 and 3).

On a GPU box an N-GPU solve is one libmadpipe call per rank: the library shards
the candidates (single chain: interleaved, madpipe_shard; batch: LPT over the
(chain, candidate) list, madpipe_batch_plan), all-reduces MIN over its own NCCL
communicator and re-solves the winners (batch: one owner per winner,
madpipe_resolve_plan, then an all-gather).  Here the same host-side plans come
from the library's host-only helpers, each rank evaluates its share with the
CPU oracle, and gloo carries the MIN all-reduce and the gather.  Every rank must
obtain the world-1 answer, every unit of work must be done exactly once, and the
bootstrap (distributed.share_id) must hand every rank the same NCCL id."""
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

INT32_MAX = 2 ** 31 - 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _run(fn, world, *args):
    with tmp.Manager() as mgr:
        out = mgr.dict()
        tmp.spawn(fn, args=(world, _free_port(), *args, out), nprocs=world, join=True)
        return dict(out)


# ------------------------------------------------------------------ bootstrap
def _id_worker(rank, world, port, out):
    _init(rank, world, port)
    from paper_conf_ipps_beaumontes22_b200 import distributed
    out[rank] = distributed.share_id()
    dist.barrier()
    dist.destroy_process_group()


def test_share_id_gives_every_rank_the_same_nccl_id():
    res = _run(_id_worker, 3)
    ids = [res[r] for r in range(3)]
    assert all(len(i) == 128 for i in ids)
    assert ids[0] == ids[1] == ids[2]


# ------------------------------------------------------------------ single chain
def _case(seed):
    rng = np.random.default_rng(seed)
    ch = chaingen.tiny(rng, 9)
    M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * (0.12 + 0.05 * seed))
    return ch, 3, M, 25.0, 4, 8, 20


def _chain_worker(rank, world, port, seed, early_exit, out):
    _init(rank, world, port)
    ch, P, M, beta, n_m, n_v, n_c = _case(seed)
    tau = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, j_lo=0, j_hi=1)["tau"]
    evaluated = []
    best = INT32_MAX
    for j in mp.shard(n_c, rank, world):                 # the library's sharding rule
        A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, 0, tau[j], with_arg=False)
        evaluated.append(j)
        if A[-1, P - 1, 0, 0] <= tau[j]:
            best = min(best, j)
            if early_exit:
                break
    jl = torch.tensor([best], dtype=torch.int32)
    dist.all_reduce(jl, op=dist.ReduceOp.MIN)            # a7
    j = int(jl.item())
    res = dict(rc=oracle.INFEASIBLE)
    if j != INT32_MAX:                                   # a8 on every rank
        r = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, j_lo=j, j_hi=j + 1)
        res = dict(rc=r["rc"], cand_index=r["cand_index"], stages=r["stages"], period=r["period"],
                   special_load=r["special_load"])
    out[rank] = (res, sorted(evaluated))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,early_exit,seed", [(2, False, 1), (2, True, 2), (3, False, 3), (3, True, 4)])
def test_chain_protocol_matches_world1(world, early_exit, seed):
    ch, P, M, beta, n_m, n_v, n_c = _case(seed)
    ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c)
    results = _run(_chain_worker, world, seed, early_exit)
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


# ------------------------------------------------------------------ batch (config 5 protocol)
def _batch(seed, n=7):
    rng = np.random.default_rng(seed)
    chains, Ps, Ms, betas = [], [], [], []
    for i in range(n):
        L = int(rng.integers(3, 9))
        ch = chaingen.tiny(rng, L, a_hi=120 if i % 2 else 40)
        chains.append(ch)
        Ps.append(int(rng.integers(1, 4)))
        Ms.append(int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * rng.uniform(0.15, 0.6)) + 1)
        betas.append(float(rng.uniform(8.0, 40.0)))
    return chains, Ps, Ms, betas, 4, 8, 12


def _batch_worker(rank, world, port, seed, early_exit, out):
    _init(rank, world, port)
    chains, Ps, Ms, betas, n_m, n_v, n_c = _batch(seed)
    n = len(chains)
    owner, load, cost = mp.batch_plan(chains, Ps, betas, n_m, n_v, n_c, world)
    # every rank must hold the same plan (it is computed, not communicated)
    plans = [None] * world
    dist.all_gather_object(plans, owner.tobytes())
    assert all(p == plans[0] for p in plans)
    taus = [oracle.solve(c, P, M, b, n_m, n_v, n_c, j_lo=0, j_hi=1)["tau"]
            for c, P, M, b in zip(chains, Ps, Ms, betas)]
    jl = np.full(n, INT32_MAX, np.int32)
    evaluated = []
    for j in range(n_c):                                 # candidate-major, as the library
        for c in range(n):
            if owner[c, j] != rank or (early_exit and jl[c] < j):
                continue
            A, _, _ = oracle.table(chains[c], Ps[c], Ms[c], betas[c], n_m, n_v, 0, taus[c][j], with_arg=False)
            evaluated.append((c, j))
            if A[-1, Ps[c] - 1, 0, 0] <= taus[c][j]:
                jl[c] = min(jl[c], j)
    t = torch.from_numpy(jl.copy())
    dist.all_reduce(t, op=dist.ReduceOp.MIN)             # a7 over int32[n]
    jstar = t.numpy()
    rown = mp.resolve_plan(chains, Ps, betas, n_m, n_v, n_c, jstar, world)
    mine = {}
    for c in range(n):
        if rown[c] == rank:
            r = oracle.solve(chains[c], Ps[c], Ms[c], betas[c], n_m, n_v, n_c, j_lo=int(jstar[c]),
                             j_hi=int(jstar[c]) + 1)
            mine[c] = (r["cand_index"], r["stages"], r["period"])
    gathered = [None] * world
    dist.all_gather_object(gathered, mine)               # the result all-gather
    allres = {}
    for g in gathered:
        assert not set(g) & set(allres)                  # each winner re-solved once
        allres.update(g)
    out[rank] = (allres, evaluated, list(jstar), list(load))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,early_exit,seed", [(2, False, 11), (3, False, 12), (3, True, 13)])
def test_batch_protocol_matches_world1(world, early_exit, seed):
    chains, Ps, Ms, betas, n_m, n_v, n_c = _batch(seed)
    refs = [oracle.solve(c, P, M, b, n_m, n_v, n_c) for c, P, M, b in zip(chains, Ps, Ms, betas)]
    results = _run(_batch_worker, world, seed, early_exit)
    evaluated = []
    for r in range(world):
        allres, ev, jstar, load = results[r]
        evaluated += ev
        for c, ref in enumerate(refs):
            if ref["rc"] != 0:
                assert jstar[c] == INT32_MAX and c not in allres
            else:
                assert jstar[c] == ref["cand_index"]
                assert allres[c] == (ref["cand_index"], ref["stages"], ref["period"])
    assert len(set(evaluated)) == len(evaluated)
    if not early_exit:
        assert sorted(evaluated) == [(c, j) for c in range(len(chains)) for j in range(n_c)]
