"""The 1F1B* simulator (O10) against the paper's statements."""
import math

import numpy as np

import chaingen
from oracle import simulator


def _contiguous(L, n, rng):
    cuts = sorted(rng.choice(np.arange(1, L), size=n - 1, replace=False)) if n > 1 else []
    bounds = [0] + [int(c) for c in cuts] + [L]
    return [(bounds[i] + 1, bounds[i + 1], i) for i in range(n)]


def test_pattern_valid_and_active_batches_equal_group():
    """P:107 (validity) and P:113 (group g stores exactly g activations) on random
    contiguous partitions at random feasible periods."""
    rng = np.random.default_rng(5)
    n_checked = 0
    for _ in range(300):
        L = int(rng.integers(2, 16))
        ch = chaingen.tiny(rng, L)
        n = int(rng.integers(1, min(L, 6) + 1))
        stages = _contiguous(L, n, rng)
        beta = float(rng.uniform(5.0, 50.0))
        loads = [sum(ch["uF"][i - 1] + ch["uB"][i - 1] for i in range(k, l + 1)) for k, l, _ in stages]
        comms = [2.0 * ch["a"][k - 1] / beta for k, _, _ in stages[1:]]
        tau = max(loads + comms) * rng.uniform(1.0, 3.0)
        P = n + 1          # the special processor stays empty
        rep = simulator.check_allocation(ch, P, 10**18, beta, tau, stages)
        assert rep["errors"] == [], rep["errors"]
        pat = rep["pattern"]
        assert pat is not None
        assert len(pat["items"]) == 2 * n - 1          # 2P-1 transformed chain
        groups = pat["group"]
        assert groups[-1] == 1 and groups == sorted(groups, reverse=True)
        n_checked += 1
    assert n_checked == 300


def test_group_count_single_group_when_period_large():
    ch = chaingen.toy()
    stages = [(1, 3, 0), (4, 6, 1), (7, 8, 2)]
    rep = simulator.check_allocation(ch, 4, 10**18, 12e9, 10.0, stages)
    assert rep["errors"] == []
    assert rep["groups"] == [1, 1, 1]
    assert all(x == 1 for x in rep["pattern"]["active"])


def test_detects_memory_violation():
    ch = chaingen.toy()
    stages = [(1, 4, 0), (5, 8, 1)]
    rep = simulator.check_allocation(ch, 3, 1, 12e9, 1.0, stages)
    assert any("needs" in e for e in rep["errors"])


def test_detects_bad_tiling_and_period():
    ch = chaingen.toy()
    rep = simulator.check_allocation(ch, 3, 10**18, 12e9, 1.0, [(1, 3, 0), (5, 8, 1)])
    assert rep["errors"]
    rep = simulator.check_allocation(ch, 3, 10**18, 12e9, 1e-6, [(1, 4, 0), (5, 8, 1)])
    assert any("exceeds tau" in e for e in rep["errors"])


def test_fig5_peaks_ordered():
    """the best-case interleaving never needs more than the worst case,
    and both are at least the (g-1) model of the DP."""
    rng = np.random.default_rng(6)
    for _ in range(100):
        L = 8
        ch = chaingen.tiny(rng, L)
        stages = [(1, 2, 3), (3, 4, 0), (5, 6, 3), (7, 8, 1)]
        rep = simulator.check_allocation(ch, 4, 10**18, 20.0, 5.0 * rng.uniform(1, 4), stages,
                                         build_pattern=False)
        assert rep["special_mem_model"] <= rep["special_peak_best"] <= rep["special_peak_worst"]
        assert not math.isnan(rep["load_period"])
