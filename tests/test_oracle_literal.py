"""NEXT row f1: the paper-literal MadPipe-DP (optimisation form, t_P discretised,
P:173-193) and Algorithm 1 in the oracle, pinned against brute force
and against the decision form."""
import math

import numpy as np

import chaingen
import oracle
from oracle import bruteforce


def _case(rng, L=None, P=None):
    L = int(rng.integers(2, 7)) if L is None else L
    P = int(rng.integers(1, 4)) if P is None else P
    ch = chaingen.tiny(rng, L)
    M = int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * rng.uniform(0.2, 0.9)) + 1
    beta = float(rng.choice([math.inf, rng.uniform(5.0, 60.0)]))
    return ch, P, M, beta, int(rng.choice([2, 4, 8])), int(rng.choice([4, 8, 16])), int(rng.choice([5, 11, 21]))


def test_literal_root_equals_bruteforce():
    rng = np.random.default_rng(61)
    n_fin = 0
    for _ in range(80):
        ch, P, M, beta, n_m, n_v, n_t = _case(rng)
        pre = oracle.prep(ch, P, beta)
        for frac in (0.0, 0.3, 0.8):
            That = pre["lb"] + frac * (pre["ub"] - pre["lb"])
            A, _ = oracle.literal_table(ch, P, M, beta, n_m, n_v, n_t, That, with_arg=False)
            bf = bruteforce.literal_root(ch, P, M, beta, n_m, n_v, n_t, That)
            assert A[-1, P - 1, 0, 0, 0] == bf
            n_fin += bf < math.inf
    assert n_fin > 60


def test_literal_feasible_implies_decision_feasible():
    """P:199 logic (reading Q1): if the literal DP at T-hat finds a period <= T-hat, the
    decision DP at tau = T-hat (same V and m grids) is feasible -- the literal form only
    rounds the special load up."""
    rng = np.random.default_rng(62)
    hits = 0
    for _ in range(60):
        ch, P, M, beta, n_m, n_v, n_t = _case(rng, L=int(rng.integers(3, 9)))
        pre = oracle.prep(ch, P, beta)
        for frac in np.linspace(0.0, 1.0, 6):
            That = pre["lb"] + frac * (pre["ub"] - pre["lb"])
            A, _ = oracle.literal_table(ch, P, M, beta, n_m, n_v, n_t, That, with_arg=False)
            if A[-1, P - 1, 0, 0, 0] <= That:
                D, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, oracle.PAPER, That, with_arg=False)
                assert D[-1, P - 1, 0, 0] <= That
                hits += 1
    assert hits > 50


def test_algorithm1_invariants():
    """Algorithm 1 (Q15): the search interval shrinks, the answer is min max(T_i, T-hat_i),
    and its allocation's literal value at the winning T-hat equals T_i."""
    rng = np.random.default_rng(63)
    for _ in range(25):
        ch, P, M, beta, n_m, n_v, n_t = _case(rng, L=int(rng.integers(3, 8)), P=int(rng.integers(2, 4)))
        r = oracle.literal_solve(ch, P, M, beta, n_m, n_v, n_t, K=10)
        pre = oracle.prep(ch, P, beta)
        assert r["That"][0] == pre["lb"]
        vals = np.maximum(r["T"], r["That"])
        if not np.isfinite(vals).any():
            assert r["rc"] == oracle.INFEASIBLE
            continue
        assert r["period"] == vals.min() and r["best_iter"] == int(np.argmin(vals))
        assert all(pre["lb"] <= th <= pre["ub"] for th in r["That"])
        i = r["best_iter"]
        c = bruteforce.Chain(ch, P, M, beta, n_m, n_v, 0)
        alloc = [((f, l), 1 if pr == P - 1 else 0) for (f, l, pr) in r["stages"]]
        val = bruteforce.literal_evaluate(c, r["That"][i], n_t, alloc, P - 1, 0, 0, 0)
        assert val == r["T"][i]


def test_golden_algorithm1_four_iterations():
    """Hand-worked Algorithm 1 (tests/golden, 'algorithm1_four_iterations'): the That_i
    sequence follows reading Q15; the printed order of P:205 would diverge at i = 2."""
    import json
    import os
    g = os.path.join(os.path.dirname(__file__), "golden", "hand_worked.json")
    ex = json.load(open(g))["examples"][3]
    beta = math.inf if ex["beta"] == "inf" else float(ex["beta"])
    r = oracle.literal_solve(ex["chain"], ex["P"], ex["M"], beta, ex["n_m"], ex["n_v"], ex["n_t"], K=ex["K"])
    e = ex["expect"]
    assert list(r["That"]) == e["That"]
    assert list(r["T"]) == e["T"]
    assert r["period"] == e["period"] and r["best_iter"] == e["best_iter"]
    assert [list(s) for s in r["stages"]] == e["stages"]
