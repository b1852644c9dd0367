"""GPU tests of the multi-GPU path on the one GPU a test box has.

* The two halves of an N-rank solve (madpipe_sweep with rank r of W, then
  madpipe_resolve of the min) run for every r in turn on one GPU; the host takes
  the min the all-reduce would take.  Result = world-1 result = oracle.
* The same for the batch (madpipe_sweep_batch / madpipe_resolve_batch, LPT plan).
* The collective code path itself: a ctx with an NCCL communicator of one rank
  (madpipe_ctx_create(rank 0, world 1, id)) runs madpipe_solve / _solve_dev /
  _solve_batch through ncclAllReduce / ncclAllGather.
* BASELINE config 5 in full: all 512 chains in one madpipe_solve_batch, every
  winner equal to the oracle's (configs/batch.json), every allocation verified by
  the 1F1B* simulator.
"""
import numpy as np
import pytest

import chaingen
import oracle
import paper_conf_ipps_beaumontes22_b200 as mp
from oracle import simulator
from paper_conf_ipps_beaumontes22_b200 import configs

pytestmark = pytest.mark.gpu
INT32_MAX = 2 ** 31 - 1


@pytest.fixture(scope="module")
def ctx():
    c = mp.Context(0)
    yield c
    c.close()


@pytest.fixture(scope="module")
def nctx():
    """A ctx with a one-rank NCCL communicator: the collective code path."""
    c = mp.Context(0, rank=0, world=1, nccl_id=mp.get_unique_id())
    assert c.info()["nccl_version"] > 0
    yield c
    c.close()


def _args(cfg):
    return (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])


def _same(got, ref):
    for key in ("rc", "cand_index", "period", "special_load", "load_period", "stages"):
        assert got[key] == ref[key], (key, got[key], ref[key])


def _verify(ch, P, M, beta, res):
    if res["rc"] != 0:
        return
    rep = simulator.check_allocation(ch, P, M, beta, res["period"], res["stages"], res["load_period"],
                                     res["special_load"], build_pattern=False)
    assert rep["errors"] == [], rep["errors"]


def _fuzz(n, seed):
    rng = np.random.default_rng(seed)
    for i in range(n):
        L = int(rng.integers(3, 16))
        ch = chaingen.tiny(rng, L, a_hi=200 if i % 2 else 40)
        P = int(rng.choice([2, 3, 6, 40]))
        M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * rng.uniform(0.2, 0.8)) + 1
        yield ch, P, M, float(rng.uniform(5.0, 40.0)), int(rng.choice([4, 8])), int(rng.choice([8, 32])), 21


def _sequential_ranks(ctx, ch, a, world, early_exit=False):
    import torch
    jl = torch.empty(1, dtype=torch.int32, device="cuda")
    best, total = INT32_MAX, 0
    for r in range(world):
        total += ctx.sweep(ch, *a, r, world, jl.data_ptr(), early_exit=early_exit)
        torch.cuda.synchronize()
        best = min(best, int(jl.item()))
    js = torch.tensor([best], dtype=torch.int32, device="cuda")
    return ctx.resolve(ch, *a, js.data_ptr()), total


@pytest.mark.parametrize("world", [2, 3, 8])
def test_sweep_ranks_then_resolve_equals_world1(ctx, world):
    cases = [(chaingen.make(configs.load(n)["chain"]), _args(configs.load(n))) for n in ("resnet50", "vgg19")]
    cases += [(ch, (P, M, b, n_m, n_v, n_c)) for ch, P, M, b, n_m, n_v, n_c in _fuzz(8, world)]
    for ch, a in cases:
        ref = ctx.solve(ch, *a)
        got, total = _sequential_ranks(ctx, ch, a, world)
        _same(got, ref)
        assert total == ref["cell_updates"]            # the shards partition the work
        ee, _ = _sequential_ranks(ctx, ch, a, world, early_exit=True)
        _same(ee, ref)


def test_nccl_world1_solve_paths(ctx, nctx):
    """madpipe_solve / _solve_dev / early_exit 1 and 2 with the ctx's communicator
    (ncclAllReduce on the ctx stream) = without it = oracle."""
    import torch
    for name in ("resnet50", "inception_v3"):
        cfg = configs.load(name)
        ch = chaingen.make(cfg["chain"])
        a = _args(cfg)
        ref = ctx.solve(ch, *a)
        assert ref["cand_index"] == cfg["oracle_cand_index"]
        _same(nctx.solve(ch, *a), ref)
        d = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).cuda() for k in ("uF", "uB", "W", "a")}
        _same(nctx.solve_dev(d, *a), ref)
        _same(nctx.solve(ch, *a, early_exit=True), ref)
        _same(nctx.solve(ch, *a, early_exit=2), ctx.solve(ch, *a, early_exit=2))
    for ch, P, M, b, n_m, n_v, n_c in _fuzz(10, 5):
        _same(nctx.solve(ch, P, M, b, n_m, n_v, n_c), oracle.solve(ch, P, M, b, n_m, n_v, n_c))


def _batch_inputs(cfg, idx):
    chains, Ps, Ms, Bs = [], [], [], []
    for i in idx:
        c = cfg["chains"][i]
        ch = chaingen.random_chain(c["seed"])
        assert chaingen.digest(ch) == c["digest"]
        chains.append(ch); Ps.append(c["P"]); Ms.append(c["M"]); Bs.append(c["beta"])
    return chains, Ps, Ms, Bs


def test_batch_config_all_512_chains(ctx):
    """BASELINE config 5 at full size: one madpipe_solve_batch over all 512 chains."""
    cfg = configs.load("batch")
    n = len(cfg["chains"])
    assert n == 512
    chains, Ps, Ms, Bs = _batch_inputs(cfg, range(n))
    res = ctx.solve_batch(chains, Ps, Ms, Bs, cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    for i, (ch, P, M, B, got) in enumerate(zip(chains, Ps, Ms, Bs, res)):
        assert got["cand_index"] == cfg["chains"][i]["oracle_cand_index"], i
        _verify(ch, P, M, B, got)
    # the oracle's full solution on a sample (the winners above are all checked)
    rng = np.random.default_rng(5)
    for i in sorted(rng.choice(n, 8, replace=False).tolist()):
        ref = oracle.solve(chains[i], Ps[i], Ms[i], Bs[i], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"],
                           early_exit=True, n_threads=8)
        _same(res[i], ref)


@pytest.mark.parametrize("world", [3, 8])
def test_batch_sweep_ranks_then_resolve_equals_world1(ctx, nctx, world):
    """The batch's N-rank protocol run rank by rank on one GPU: LPT shares
    (madpipe_sweep_batch), element-wise MIN, owner re-solves (madpipe_resolve_batch);
    and the one-rank NCCL path of madpipe_solve_batch (all-reduce + all-gather)."""
    cfg = configs.load("batch")
    idx = list(range(0, 512, 9))
    chains, Ps, Ms, Bs = _batch_inputs(cfg, idx)
    d = (cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    ref = ctx.solve_batch(chains, Ps, Ms, Bs, *d)
    owner, load, cost = mp.batch_plan(chains, Ps, Bs, *d, world)
    jmin = np.full(len(chains), INT32_MAX, np.int64)
    cu = np.zeros(len(chains), np.int64)
    for r in range(world):
        jl, c = ctx.sweep_batch(chains, Ps, Ms, Bs, *d, r, world)
        jmin = np.minimum(jmin, jl)
        cu += c
    for i, rr in enumerate(ref):
        assert jmin[i] == (rr["cand_index"] if rr["cand_index"] >= 0 else INT32_MAX), i
        assert cu[i] == rr["cell_updates"], i
    got = {}
    for r in range(world):
        part = ctx.resolve_batch(chains, Ps, Ms, Bs, *d, jmin.astype(np.int32), r, world)
        assert not set(part) & set(got)
        got.update(part)
    for i, rr in enumerate(ref):
        if rr["cand_index"] >= 0:
            _same(got[i], rr)
        else:
            assert i not in got
    for g, rr in zip(nctx.solve_batch(chains, Ps, Ms, Bs, *d), ref):
        _same(g, rr)


def test_fig6_sweep_batch_matches_oracle(ctx):
    """NEXT row f4 (scripts/fig6_sweep.py): the 84 Fig. 6-style instances -- ResNet-50-shaped
    chain, M = 3..16 GB x P in {2, 4, 8} x beta in {12, 24} GB/s, the paper's 11 x 51
    discretisation -- in one madpipe_solve_batch, each equal to the oracle."""
    ch = chaingen.resnet50()
    inst = [(g * 10**9, P, b) for b in (12e9, 24e9) for P in (2, 4, 8) for g in range(3, 17)]
    n_c = 48
    res = ctx.solve_batch([ch] * len(inst), [P for _, P, _ in inst], [M for M, _, _ in inst],
                          [b for _, _, b in inst], 11, 51, n_c)
    for (M, P, b), got in zip(inst, res):
        ref = oracle.solve(ch, P, M, b, 11, 51, n_c, early_exit=True, n_threads=8)
        _same(got, ref)
        _verify(ch, P, M, b, got)
