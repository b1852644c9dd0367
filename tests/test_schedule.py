"""NEXT row f2: madpipe_schedule (product, host-only C ABI) against the oracle's 1F1B*
simulator on random contiguous allocations."""
import math

import numpy as np

import chaingen
import paper_conf_ipps_beaumontes22_b200 as mp
from oracle import simulator


def _contiguous(L, n, rng):
    cuts = sorted(rng.choice(np.arange(1, L), size=n - 1, replace=False)) if n > 1 else []
    b = [0] + [int(c) for c in cuts] + [L]
    return [(b[i] + 1, b[i + 1], i) for i in range(n)]


def test_schedule_matches_simulator():
    rng = np.random.default_rng(9)
    for _ in range(300):
        L = int(rng.integers(1, 20))
        ch = chaingen.tiny(rng, L)
        n = int(rng.integers(1, min(L, 7) + 1))
        stages = _contiguous(L, n, rng)
        beta = float(rng.uniform(5.0, 50.0))
        loads = [sum(ch["uF"][i - 1] + ch["uB"][i - 1] for i in range(k, l + 1)) for k, l, _ in stages]
        comms = [2.0 * ch["a"][k - 1] / beta for k, _, _ in stages[1:]]
        tau = max(loads + comms) * rng.uniform(1.0, 3.0)
        rep = simulator.check_allocation(ch, n + 1, 10**18, beta, tau, stages)
        assert rep["errors"] == []
        ref = rep["pattern"]
        got = mp.schedule(ch, beta, tau, stages)
        assert len(got) == 2 * n - 1
        for o, (kind, idx), g, pat in zip(got, ref["items"], ref["group"], ref["pattern"]):
            assert o["kind"] == kind and o["stage"] == idx and o["group"] == g
            assert o["F"][1] == pat["F"][1] and o["B"][1] == pat["B"][1]
            assert math.isclose(o["F"][0], pat["F"][0], rel_tol=1e-12, abs_tol=1e-15 * tau)
            assert math.isclose(o["B"][0], pat["B"][0], rel_tol=1e-12, abs_tol=1e-15 * tau)
        # active batches of every stage = its group index
        for o, act, g in zip(got, ref["active"], ref["group"]):
            assert act == g


def test_schedule_rejects_bad_input():
    ch = chaingen.toy()
    assert mp.schedule(ch, 12e9, 1e-9, [(1, 4, 0), (5, 8, 1)]) is None       # item > period
    try:
        mp.schedule(ch, 12e9, 1.0, [(1, 3, 0), (5, 8, 1)])
        assert False
    except mp.MadpipeError as e:
        assert e.rc == -1
