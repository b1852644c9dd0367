"""The C-ABI library without a GPU: it builds for sm_100a, loads, exports every
symbol include/madpipe.h declares, and its host-only helpers behave as the header
states.  No compute call is made here."""
import math
import os
import re

import numpy as np
import pytest

import chaingen
import oracle
import paper_conf_ipps_beaumontes22_b200 as mp
from paper_conf_ipps_beaumontes22_b200 import _native as N

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "madpipe.h")


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_ipps_beaumontes22_b200 import build
    build.build()
    return N.lib()


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(madpipe_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol():
    names = declared_functions()
    assert len(names) >= 15
    lib = N.lib()
    for n in names:
        assert hasattr(lib, n), n
    assert sorted(N.EXPORTED) == names


def test_sass_is_sm100a():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", N.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _disc():
    return dict(n_mem=8, n_delay=16, n_periods=8)


def test_validate_rules():
    ch = chaingen.toy()
    good = dict(chain=ch, P=2, M=10**9, beta=12e9, **_disc())
    assert mp.validate(**good) == 0
    assert mp.validate(**{**good, "beta": math.inf}) == 0
    bad_cases = [dict(P=0), dict(M=0), dict(beta=0.0), dict(beta=float("nan")), dict(n_mem=1),
                 dict(n_mem=65), dict(n_delay=1), dict(n_periods=0), dict(v_range=2)]
    for b in bad_cases:
        assert mp.validate(**{**good, **b}) == N.EINVAL, b
    for key, val in [("uF", -1.0), ("uB", float("inf")), ("W", -5)]:
        c2 = {k: np.array(v, copy=True) for k, v in ch.items() if k != "name"}
        c2[key][3] = val
        assert mp.validate(**{**good, "chain": c2}) == N.EINVAL, key
    c2 = {k: np.array(v, copy=True) for k, v in ch.items() if k != "name"}
    c2["uF"][0] = 0.0; c2["uB"][0] = 0.0          # uF+uB = 0 (reading Q9)
    assert mp.validate(**{**good, "chain": c2}) == N.EINVAL
    c2 = {k: np.array(v, copy=True) for k, v in ch.items() if k != "name"}
    c2["a"][5] = -1
    assert mp.validate(**{**good, "chain": c2}) == N.EINVAL
    # int64 overflow guard
    c2 = {k: np.array(v, copy=True) for k, v in ch.items() if k != "name"}
    c2["a"][:] = 10**17
    assert mp.validate(**{**good, "chain": c2}) == N.EINVAL


def test_shard_covers_each_candidate_once():
    for n_c in (1, 7, 32, 1024, 1023):
        for world in (1, 2, 3, 4, 8):
            seen = []
            for r in range(world):
                own = mp.shard(n_c, r, world)
                assert own == sorted(own)
                assert all(j % world == r for j in own)
                seen += own
            assert sorted(seen) == list(range(n_c))


def test_cell_update_count_matches_oracle():
    rng = np.random.default_rng(3)
    for _ in range(20):
        L = int(rng.integers(2, 30))
        ch = chaingen.tiny(rng, L)
        P = int(rng.integers(1, 6))
        pre = oracle.prep(ch, P, 20.0)
        tau = pre["lb"] + rng.uniform(0, 1) * (pre["ub"] - pre["lb"])
        _, _, cu = oracle.table(ch, P, 10**9, 20.0, 2, 2, 0, tau, with_arg=False)
        assert mp.cell_updates(ch, P, 2, 2, tau) == cu


def test_no_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(mp.MadpipeError) as e:
        mp.Context(0)
    assert e.value.rc == N.ECUDA


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_beaumontes22_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle", src, re.M), f
                assert "madpipe_oracle" not in src, f


def _plan_batch(seed, n=12):
    rng = np.random.default_rng(seed)
    chains = [chaingen.tiny(rng, int(rng.integers(2, 40))) for _ in range(n)]
    Ps = [int(rng.integers(1, 9)) for _ in range(n)]
    betas = [float(rng.uniform(5, 50)) for _ in range(n)]
    return chains, Ps, betas


def test_batch_plan_lpt():
    """madpipe_batch_plan: every (chain, candidate) pair has exactly one
    owner, the cost of a pair is its exact cell-update count plus the fixed row work,
    the plan is deterministic, and LPT keeps the ranks within one largest job."""
    chains, Ps, betas = _plan_batch(5)
    n_m, n_v, n_c = 4, 8, 16
    for world in (1, 2, 3, 8):
        owner, load, cost = mp.batch_plan(chains, Ps, betas, n_m, n_v, n_c, world)
        owner2, load2, _ = mp.batch_plan(chains, Ps, betas, n_m, n_v, n_c, world)
        assert np.array_equal(owner, owner2) and np.array_equal(load, load2)
        assert owner.min() >= 0 and owner.max() < world
        for r in range(world):
            assert load[r] == cost[owner == r].sum()
        assert load.sum() == cost.sum()
        assert load.max() - load.min() <= cost.max()
    for c, (ch, P, b) in enumerate(zip(chains, Ps, betas)):
        pre = oracle.prep(ch, P, b)
        for j in (0, 7, 15):
            tau = pre["lb"] + j * ((pre["ub"] - pre["lb"]) / (n_c - 1))
            L = len(ch["uF"])
            assert cost[c, j] == mp.cell_updates(ch, P, n_m, n_v, tau) + (L + 1) * n_v * P


def test_resolve_plan_one_owner_per_winner():
    chains, Ps, betas = _plan_batch(6)
    jstar = np.array([c % 16 if c % 3 else 2 ** 31 - 1 for c in range(len(chains))], np.int32)
    for world in (1, 2, 5):
        own = mp.resolve_plan(chains, Ps, betas, 4, 8, 16, jstar, world)
        for c in range(len(chains)):
            if jstar[c] == 2 ** 31 - 1:
                assert own[c] == -1
            else:
                assert 0 <= own[c] < world


def test_nccl_unique_id_on_cpu():
    """madpipe_get_unique_id needs only libnccl (dlopen'ed), not a GPU."""
    a = mp.get_unique_id()
    b = mp.get_unique_id()
    assert len(a) == 128 and a != b


def test_ctx_create_rejects_bad_rank_world():
    for rank, world, nid in [(0, 0, None), (2, 2, b"\0" * 128), (-1, 2, b"\0" * 128), (1, 2, None)]:
        with pytest.raises(mp.MadpipeError) as e:
            mp.Context(0, rank=rank, world=world, nccl_id=nid)
        assert e.value.rc == N.EINVAL
