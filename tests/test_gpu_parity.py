"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, on the same
seeded inputs.  Bar (BASELINE.json north_star): bit-exact fp64 DP values, decisions,
candidate periods and allocations; the 1F1B* simulator verifies every returned
allocation (period within 1e-12 relative, memory <= M)."""
import math

import numpy as np
import pytest

import chaingen
import oracle
import paper_conf_ipps_beaumontes22_b200 as mp
from oracle import simulator
from paper_conf_ipps_beaumontes22_b200 import configs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    import torch
    assert torch.cuda.is_available()
    c = mp.Context(0)
    yield c
    c.close()


def _ctx_with_kernel(kernel):
    """A context whose step kernel is forced (MADPIPE_KERNEL is read at creation)."""
    import os
    old = os.environ.get("MADPIPE_KERNEL")
    os.environ["MADPIPE_KERNEL"] = kernel
    try:
        return mp.Context(0)
    finally:
        if old is None:
            del os.environ["MADPIPE_KERNEL"]
        else:
            os.environ["MADPIPE_KERNEL"] = old


@pytest.fixture(scope="module", params=["pair", "persist", "v1"])
def kctx(request):
    c = _ctx_with_kernel(request.param)
    yield c
    c.close()


def _args(cfg):
    return (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])


def _same_solution(got, ref):
    for key in ("rc", "cand_index", "period", "special_load", "load_period", "stages"):
        assert got[key] == ref[key], (key, got[key], ref[key])


def _verify(ch, P, M, beta, res):
    if res["rc"] != 0:
        return
    rep = simulator.check_allocation(ch, P, M, beta, res["period"], res["stages"],
                                     res["load_period"], res["special_load"])
    assert rep["errors"] == [], rep["errors"]


# ---------------------------------------------------------------- toy: everything, every candidate
def test_toy_full_tables_every_candidate(kctx):
    ctx = kctx
    cfg = configs.load("toy")
    ch = chaingen.make(cfg["chain"])
    a = _args(cfg)
    ref = oracle.solve(ch, *a)
    tau, root = ctx.candidates(ch, *a)
    assert np.array_equal(tau, ref["tau"]) and np.array_equal(root, ref["root"])
    for j in range(cfg["n_periods"]):
        A, ARG = ctx.dp_table(ch, *a, j=j)
        A_ref, ARG_ref, _ = oracle.table(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"],
                                         cfg["n_delay"], 0, ref["tau"][j])
        assert np.array_equal(A, A_ref), j
        assert np.array_equal(ARG, ARG_ref), j
    got = ctx.solve(ch, *a)
    _same_solution(got, ref)
    assert got["cell_updates"] == ref["cell_updates"]
    _verify(ch, cfg["P"], cfg["M"], cfg["beta"], got)


# ---------------------------------------------------------------- fuzz: tiny chains, all features
def _fuzz_cases(n, seed):
    rng = np.random.default_rng(seed)
    for i in range(n):
        L = int(rng.integers(1, 14))
        P = int(rng.integers(1, 7))
        ch = chaingen.tiny(rng, L, integer_times=bool(i % 3 == 0), zero_mem=bool(i % 7 == 0))
        n_m = int(rng.choice([2, 3, 4, 8, 11, 16, 33]))
        n_v = int(rng.choice([2, 5, 16, 51, 100]))
        n_c = int(rng.choice([1, 3, 17]))
        vr = int(rng.integers(0, 2))
        mem = 3 * int(ch["W"].sum()) + 3 * int(ch["a"].sum()) + 1
        M = int(mem * rng.uniform(0.1, 1.0)) + 1
        beta = float(rng.choice([math.inf, rng.uniform(5.0, 60.0)]))
        yield ch, P, M, beta, n_m, n_v, n_c, vr


def test_fuzz_roots_tables_solutions(kctx):
    ctx = kctx
    for ch, P, M, beta, n_m, n_v, n_c, vr in _fuzz_cases(120, 7):
        ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        tau, root = ctx.candidates(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        assert np.array_equal(tau, ref["tau"])
        assert np.array_equal(root, ref["root"]), (P, n_m, n_v, vr)
        got = ctx.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        _same_solution(got, ref)
        assert got["cell_updates"] == ref["cell_updates"]
        j = max(ref["cand_index"], 0)
        A, ARG = ctx.dp_table(ch, P, M, beta, n_m, n_v, n_c, j=j, v_range=vr)
        A_ref, ARG_ref, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, ref["tau"][j])
        assert np.array_equal(A, A_ref) and np.array_equal(ARG, ARG_ref)
        _verify(ch, P, M, beta, got)


def test_early_exit_same_answer(ctx):
    for ch, P, M, beta, n_m, n_v, n_c, vr in _fuzz_cases(30, 8):
        full = ctx.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        ee = ctx.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, early_exit=True)
        _same_solution(ee, full)
        assert ee["cell_updates"] <= full["cell_updates"]


def test_paper_discretisation(ctx):
    """The paper's own grid: 11 memory levels, 51 delay levels."""
    ch = chaingen.resnet50()
    a = (4, 8 * 10**9, 12e9, 11, 51, 16)
    ref = oracle.solve(ch, *a, n_threads=8)
    got = ctx.solve(ch, *a)
    _same_solution(got, ref)
    tau, root = ctx.candidates(ch, *a)
    assert np.array_equal(root, ref["root"])


# ---------------------------------------------------------------- BASELINE configs
def _sampled(ref_tau, jstar, n_c, extra_hi=4):
    js = set(range(0, min(jstar + 3, n_c)))
    hi = np.linspace(jstar + 3, n_c - 1, extra_hi).astype(int) if jstar + 3 < n_c else []
    js.update(int(x) for x in hi)
    return sorted(js)


@pytest.mark.parametrize("name", ["resnet50", "inception_v3", "vgg19"])
def test_cnn_configs(ctx, name):
    cfg = configs.load(name)
    ch = chaingen.make(cfg["chain"])
    assert chaingen.digest(ch) == cfg["digest"]
    a = _args(cfg)
    got = ctx.solve(ch, *a)
    assert got["cand_index"] == cfg["oracle_cand_index"]
    ref = oracle.solve(ch, *a, early_exit=True, n_threads=8)
    _same_solution(got, ref)
    tau, root = ctx.candidates(ch, *a)
    assert np.array_equal(tau, ref["tau"])
    for j in _sampled(ref["tau"], ref["cand_index"], cfg["n_periods"]):
        A_ref, _, _ = oracle.table(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"],
                                   cfg["n_delay"], 0, tau[j], with_arg=False)
        assert root[j] == A_ref[-1, cfg["P"] - 1, 0, 0], j
    # full table and decisions of the winner
    j = got["cand_index"]
    A, ARG = ctx.dp_table(ch, *a, j=j)
    A_ref, ARG_ref, _ = oracle.table(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"],
                                     cfg["n_delay"], 0, tau[j])
    assert np.array_equal(A, A_ref) and np.array_equal(ARG, ARG_ref)
    _verify(ch, cfg["P"], cfg["M"], cfg["beta"], got)


def test_gpt_config_sampled(ctx):
    """Full BASELINE size, bench launch configuration: the solve, the winner and a
    sample of candidate roots (cheap low periods + stratified high ones)."""
    cfg = configs.load("gpt")
    ch = chaingen.make(cfg["chain"])
    assert chaingen.digest(ch) == cfg["digest"]
    a = _args(cfg)
    got = ctx.solve(ch, *a)
    assert got["cand_index"] == cfg["oracle_cand_index"]
    ref = oracle.solve(ch, *a, early_exit=True, n_threads=8)
    _same_solution(got, ref)
    _verify(ch, cfg["P"], cfg["M"], cfg["beta"], got)
    ee = ctx.solve(ch, *a, early_exit=True)
    _same_solution(ee, ref)
    tau, root = ctx.candidates(ch, *a)
    assert np.array_equal(tau, ref["tau"])
    jstar = ref["cand_index"]
    for j in [0, max(0, jstar - 1), jstar, min(jstar + 1, 1023), 300]:
        A_ref, _, _ = oracle.table(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"],
                                   cfg["n_delay"], 0, tau[j], with_arg=False)
        assert root[j] == A_ref[-1, cfg["P"] - 1, 0, 0], j


def test_batch_config_sampled(ctx):
    cfg = configs.load("batch")
    rng = np.random.default_rng(0)
    pick = sorted(rng.choice(len(cfg["chains"]), size=24, replace=False).tolist())
    chains, Ps, Ms, Bs = [], [], [], []
    for i in pick:
        c = cfg["chains"][i]
        ch = chaingen.random_chain(c["seed"])
        assert chaingen.digest(ch) == c["digest"]
        chains.append(ch); Ps.append(c["P"]); Ms.append(c["M"]); Bs.append(c["beta"])
    res = ctx.solve_batch(chains, Ps, Ms, Bs, cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    for i, ch, P, M, B, got in zip(pick, chains, Ps, Ms, Bs, res):
        ref = oracle.solve(ch, P, M, B, cfg["n_mem"], cfg["n_delay"], cfg["n_periods"],
                           early_exit=True, n_threads=8)
        _same_solution(got, ref)
        assert got["cand_index"] == cfg["chains"][i]["oracle_cand_index"]
        _verify(ch, P, M, B, got)


def test_coarse_to_fine_matches_full_sweep_when_monotone(ctx):
    """NEXT row f3 (early_exit=2): equal to the full sweep whenever feasibility is monotone
    in the period; checked on fuzz cases and on the CNN configs."""
    n_checked = 0
    for ch, P, M, beta, n_m, n_v, n_c, vr in _fuzz_cases(60, 10):
        n_c = 40
        tau, root = ctx.candidates(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        feas = [root[j] <= tau[j] for j in range(n_c)]
        if any(feas[j] and not feas[j + 1] for j in range(n_c - 1)):
            continue            # not monotone: f3 is allowed to differ
        full = ctx.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        ctf = ctx.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, early_exit=2)
        _same_solution(ctf, full)
        n_checked += 1
    assert n_checked > 30
    for name in ("resnet50", "vgg19"):
        cfg = configs.load(name)
        ch = chaingen.make(cfg["chain"])
        full = ctx.solve(ch, *_args(cfg), early_exit=True)
        ctf = ctx.solve(ch, *_args(cfg), early_exit=2)
        _same_solution(ctf, full)
        assert ctf["cell_updates"] <= full["cell_updates"] * 2


@pytest.mark.parametrize("P,n_m,n_v,L", [(300, 4, 6, 9),      # ROW mode, 2 processor tiles
                                         (40, 33, 5, 8),      # PAIR mode (NMP 64), 5 processor tiles
                                         (20, 17, 4, 10),     # PAIR mode (NMP 32), 2 processor tiles
                                         (5, 8, 300, 12),     # delay levels above 255
                                         (1, 8, 16, 30),      # P = 1: base rows only
                                         (3, 2, 2, 1)])       # L = 1, smallest grids
def test_geometry_extremes(P, n_m, n_v, L):
    """Tile geometries the configs do not reach (processor tiling, wide delay grids,
    P = 1, L = 1), for every step kernel, against the oracle."""
    rng = np.random.default_rng(P * 1000 + n_m)
    ch = chaingen.tiny(rng, L)
    M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * 0.6) + 1
    n_c = 9
    ref = oracle.solve(ch, P, M, 25.0, n_m, n_v, n_c, v_range=1, n_threads=4)
    for kernel in ("pair", "persist", "v1"):
        c = _ctx_with_kernel(kernel)
        try:
            tau, root = c.candidates(ch, P, M, 25.0, n_m, n_v, n_c, v_range=1)
            assert np.array_equal(root, ref["root"]), kernel
            got = c.solve(ch, P, M, 25.0, n_m, n_v, n_c, v_range=1)
            _same_solution(got, ref)
        finally:
            c.close()


@pytest.mark.parametrize("seed,P,n_m,n_v,L", [(11, 64, 8, 96, 24),    # 2 processor rows per thread
                                              (12, 40, 4, 130, 18),   # ragged v-tiles, nmp 4
                                              (13, 90, 8, 40, 15),    # 2 processor tiles (64 + 25)
                                              (14, 33, 5, 200, 21)])  # odd n_m, one row past 32
def test_two_layer_kernel_full_tables(seed, P, n_m, n_v, L):
    """The two-layer step kernel (shared source rows, layer-(l+1) shift, the k = l+1
    fixup) against the oracle's full tables, several candidates, both v ranges."""
    rng = np.random.default_rng(seed)
    ch = chaingen.tiny(rng, L)
    M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * 0.5) + 1
    n_c = 6
    c = _ctx_with_kernel("pair")
    try:
        for vr in (0, 1):
            ref = oracle.solve(ch, P, M, 30.0, n_m, n_v, n_c, v_range=vr, n_threads=4)
            tau, root = c.candidates(ch, P, M, 30.0, n_m, n_v, n_c, v_range=vr)
            assert np.array_equal(tau, ref["tau"]) and np.array_equal(root, ref["root"]), vr
            for j in (0, n_c // 2, n_c - 1):
                A, ARG = c.dp_table(ch, P, M, 30.0, n_m, n_v, n_c, j=j, v_range=vr)
                A_ref, ARG_ref, _ = oracle.table(ch, P, M, 30.0, n_m, n_v, vr, ref["tau"][j])
                assert np.array_equal(A, A_ref), (vr, j)
                assert np.array_equal(ARG, ARG_ref), (vr, j)
            got = c.solve(ch, P, M, 30.0, n_m, n_v, n_c, v_range=vr)
            _same_solution(got, ref)
            sb = c.last_step_bytes()
            assert sb["segments"] > 0 and sb["load_bytes"] > 0
    finally:
        c.close()


@pytest.mark.parametrize("kernel", ["pair", "persist", "v1"])
def test_batch_mixed_lengths(kernel):
    """One solve_batch over chains of different lengths and one P (they share a
    launch): passes beyond a chain's L must leave its table alone, for every step
    kernel; each chain's solution equals the oracle's."""
    rng = np.random.default_rng(77)
    Ls = [9, 23, 4, 16, 31, 12]
    chains = [chaingen.tiny(rng, L) for L in Ls]
    P, n_m, n_v, n_c = 40, 8, 48, 7
    Ms = [int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * 0.5) + 1 for ch in chains]
    Bs = [30.0] * len(chains)
    c = _ctx_with_kernel(kernel)
    try:
        res = c.solve_batch(chains, [P] * len(chains), Ms, Bs, n_m, n_v, n_c, v_range=1)
    finally:
        c.close()
    for ch, M, got in zip(chains, Ms, res):
        ref = oracle.solve(ch, P, M, 30.0, n_m, n_v, n_c, v_range=1, n_threads=4)
        _same_solution(got, ref)


def test_work_counters_agree_across_kernels():
    """The live-relaxation counter (madpipe_last_counts: effective_updates) is a property
    of the DP instance, not of the kernel: the two-layer path (counted by its trans and
    fixup kernels) must report the same count as the one-layer kernels.  The useful count
    (live and reading a finite source row) is kept by the persistent kernels only and is
    bounded by the effective count."""
    rng = np.random.default_rng(21)
    ch = chaingen.tiny(rng, 20)
    P, n_m, n_v, n_c = 48, 8, 96, 5
    M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * 0.5) + 1
    counts = {}
    for kernel in ("pair", "persist", "v1"):
        c = _ctx_with_kernel(kernel)
        try:
            c.solve(ch, P, M, 30.0, n_m, n_v, n_c, v_range=1)
            counts[kernel] = c.last_counts()
        finally:
            c.close()
    for kernel, got in counts.items():
        assert got["cell_updates"] == counts["v1"]["cell_updates"], kernel
        assert got["effective_updates"] == counts["v1"]["effective_updates"], (kernel, counts)
        assert got["useful_updates"] <= got["effective_updates"], (kernel, got)
        if kernel != "v1":
            assert got["useful_updates"] > 0, (kernel, got)


# ---------------------------------------------------------------- communication-bound chains
def _comm_cases(n, seed):
    """Two boundaries with activations of 200-400 bytes and beta in [5, 30] (C(i) =
    2 a_i / beta far above the stage loads, while sum C stays small enough that the
    uniform candidate grid on [lb, ub] spends about a third of its periods below
    max C): C(k-1) > tau prunes splits and links bound the allocation
    period."""
    rng = np.random.default_rng(seed)
    for i in range(n):
        L = int(rng.integers(4, 20))
        P = int(rng.choice([2, 3, 5, 9, 34, 40, 70]))
        ch = chaingen.tiny(rng, L)
        hv = rng.choice(np.arange(1, L), size=min(2, L - 1), replace=False)
        ch["a"][hv] = rng.integers(200, 400, size=len(hv))
        n_m = int(rng.choice([3, 4, 5, 8]))
        n_v = int(rng.choice([5, 16, 51]))
        vr = int(rng.integers(0, 2))
        mem = 3 * int(ch["W"].sum()) + 3 * int(ch["a"].sum()) + 1
        M = int(mem * rng.uniform(0.15, 0.9)) + 1
        beta = float(rng.uniform(5.0, 30.0))
        yield ch, P, M, beta, n_m, n_v, 24, vr


def test_comm_heavy_every_kernel(kctx):
    ctx = kctx
    pairs = with_c = 0
    for ch, P, M, beta, n_m, n_v, n_c, vr in _comm_cases(40, 91):
        ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, n_threads=4)
        tau, root = ctx.candidates(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        assert np.array_equal(tau, ref["tau"]) and np.array_equal(root, ref["root"]), (P, n_m, n_v, vr)
        got = ctx.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        _same_solution(got, ref)
        j = max(ref["cand_index"], 0)
        A, ARG = ctx.dp_table(ch, P, M, beta, n_m, n_v, n_c, j=j, v_range=vr)
        A_ref, ARG_ref, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, ref["tau"][j])
        assert np.array_equal(A, A_ref) and np.array_equal(ARG, ARG_ref)
        _verify(ch, P, M, beta, got)
        cmax = max(2.0 * ch["a"][i] / beta for i in range(1, len(ch["uF"]))) if len(ch["uF"]) > 1 else 0.0
        pairs += n_c
        with_c += int(sum(cmax > t for t in tau))
    assert with_c >= 0.25 * pairs, (with_c, pairs)


# ---------------------------------------------------------------- GPT: stratified high periods
def test_gpt_stratified_candidates_and_slabs(ctx):
    """SURVEY.md 8(d)'s GPT sample (j <= j*, j*+1..8, 16 stratified above, 511/767/1023)
    at full size: every candidate's root, and two whole table slabs (l = L/2, l = L) of
    each sampled candidate, against values written by scripts/oracle_gpt_samples.py."""
    import hashlib
    cfg = configs.load("gpt")
    sam = configs.load("gpt_oracle_samples")
    assert sam["digest"] == cfg["digest"]
    ch = chaingen.make(cfg["chain"])
    a = _args(cfg)
    tau, root = ctx.candidates(ch, *a)
    L = cfg["L"]
    assert len(sam["samples"]) >= 30
    for s in sam["samples"]:
        j = s["j"]
        assert tau[j] == float.fromhex(s["tau"]), j
        assert root[j] == float.fromhex(s["root"]), j
        A, _ = ctx.dp_table(ch, *a, j=j, with_arg=False)
        for l, dg in s["slab_sha256"].items():
            assert hashlib.sha256(np.ascontiguousarray(A[int(l)]).tobytes()).hexdigest() == dg, (j, l)
    assert max(s["j"] for s in sam["samples"]) == cfg["n_periods"] - 1


def test_solve_dev_equals_solve_equals_oracle(ctx):
    """madpipe_solve_dev (the entry bench.py times) on device-resident chains gives the
    same result as madpipe_solve on host arrays, and as the oracle."""
    import torch
    for name in ("gpt", "resnet50"):
        cfg = configs.load(name)
        ch = chaingen.make(cfg["chain"])
        a = _args(cfg)
        d = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).cuda() for k in ("uF", "uB", "W", "a")}
        dev = ctx.solve_dev(d, *a)
        host = ctx.solve(ch, *a)
        _same_solution(dev, host)
        assert dev["cell_updates"] == host["cell_updates"]
        assert dev["cand_index"] == cfg["oracle_cand_index"]
        ref = oracle.solve(ch, *a, early_exit=True, n_threads=8)
        _same_solution(dev, ref)
    for ch, P, M, beta, n_m, n_v, n_c, vr in _fuzz_cases(10, 31):
        d = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).cuda() for k in ("uF", "uB", "W", "a")}
        ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
        _same_solution(ctx.solve_dev(d, P, M, beta, n_m, n_v, n_c, v_range=vr), ref)


@pytest.mark.parametrize("env", [{"MADPIPE_TRANS_OVERLAP": "1"}, {"MADPIPE_TRANS_OVERLAP": "2"},
                                 {"MADPIPE_AUX_GRID": "4,3"}, {"MADPIPE_PAIR_ROUND": "1"},
                                 {"MADPIPE_PAIR_ROUND": "16"}])
def test_pair_schedules(env, monkeypatch):
    """The two-layer path's alternative schedules -- list building vs step and fixup (lists
    of pass i+1 beside step(i) with unverified sources; after the fixup on one stream;
    persistent list-builder / fixup grids) and the producer's round size (one slot per
    round: the queue protocol at its finest grain; 16 slots: most of the ring in flight) --
    give the oracle's roots, tables and solutions."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)                 # read at context creation or at every launch
    monkeypatch.setenv("MADPIPE_KERNEL", "pair")
    c = mp.Context(0)
    try:
        for ch, P, M, beta, n_m, n_v, n_c, vr in _comm_cases(6, 123):
            ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, n_threads=4)
            tau, root = c.candidates(ch, P, M, beta, n_m, n_v, n_c, v_range=vr)
            assert np.array_equal(root, ref["root"]), (P, n_m, n_v, vr)
            _same_solution(c.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr), ref)
            j = max(ref["cand_index"], 0)
            A, _ = c.dp_table(ch, P, M, beta, n_m, n_v, n_c, j=j, v_range=vr)
            A_ref, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, ref["tau"][j])
            assert np.array_equal(A, A_ref)
        cfg = configs.load("resnet50")
        ch = chaingen.make(cfg["chain"])
        got = c.solve(ch, *_args(cfg))
        assert got["cand_index"] == cfg["oracle_cand_index"]
    finally:
        c.close()


@pytest.mark.parametrize("kernel", ["pair", "persist", "v1"])
def test_winner_traced_in_a_later_batch(kernel, monkeypatch):
    """One-rank solves trace the winner straight from the sweep batch that found it (no
    re-solve).  A table budget of one job per batch puts the winner in a later batch than the
    first, for the full sweep and for early exit; allocations equal the oracle's and pass
    the simulator, and the single-batch context agrees."""
    monkeypatch.setenv("MADPIPE_KERNEL", kernel)
    tiny = mp.Context(0, mem_budget=1)            # every batch: a single job
    big = mp.Context(0)
    try:
        n_checked = 0
        for ch, P, M, beta, n_m, n_v, n_c, vr in _comm_cases(12, 321):
            ref = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, n_threads=4)
            if ref["rc"] != 0 or ref["cand_index"] < 1:
                continue
            for early in (False, True):
                got = tiny.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, early_exit=early)
                _same_solution(got, ref)
                _verify(ch, P, M, beta, got)
                _same_solution(big.solve(ch, P, M, beta, n_m, n_v, n_c, v_range=vr, early_exit=early), ref)
            n_checked += 1
        assert n_checked >= 3, n_checked
    finally:
        tiny.close()
        big.close()
