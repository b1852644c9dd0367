"""Pins of the CPU oracle against things other than itself.

Each test names what fixes the expected value: a hand-worked example
(tests/golden), a closed form, an independent algorithm (brute force over all
allocations, 1F1B* grouping, max-coverage DP) or an invariant.
"""
import json
import math
import os

import numpy as np
import pytest

import chaingen
import oracle
from oracle import bruteforce, simulator, special

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hand_worked.json")
INF = math.inf


def _beta(x):
    return math.inf if x == "inf" else float(x)


# ------------------------------------------------------------------ O1 / O2 / O3 closed forms
def test_prefix_sums_and_bounds_hand():
    """P:155 U(k,l), P:147 C(l) = 2 a_l / beta, P:205 lb = U(1,L)/P, ub = U(1,L) + sum C (Q4)."""
    ch = {"uF": [1.0, 2.0, 3.0], "uB": [2.0, 4.0, 6.0], "W": [5, 6, 7], "a": [10, 20, 30, 40]}
    r = oracle.prep(ch, P=3, beta=10.0)
    assert list(r["Up"]) == [0.0, 3.0, 9.0, 18.0]
    assert list(r["Wp"]) == [0, 5, 11, 18]
    assert list(r["Ap"]) == [0, 10, 30, 60]          # sums of a_{i-1}
    assert list(r["C"][:3]) == [0.0, 4.0, 6.0]       # C(1)=2*20/10, C(2)=2*30/10; no C(3)
    assert r["SC"] == 10.0
    assert r["lb"] == 6.0 and r["ub"] == 28.0


def test_mem_hand_cases():
    """M(k,l,g) = sum(3W_i + g a_{i-1}) + 2(a_{k-1} + a_l), buffer terms dropped at k=1 / l=L."""
    W = [5, 6, 7]
    a = [10, 20, 30, 40]
    assert oracle.mem(W, a, 1, 3, 2) == 3 * 18 + 2 * 60                # no buffers at all
    assert oracle.mem(W, a, 2, 2, 1) == 3 * 6 + 20 + 2 * (20 + 30)    # both buffers
    assert oracle.mem(W, a, 1, 1, 3) == 15 + 3 * 10 + 2 * 20          # only a_l buffer
    assert oracle.mem(W, a, 3, 3, 0) == 21 + 2 * 30                   # only a_{k-1} buffer
    g = json.load(open(GOLD))["examples"][1]
    for (k, l, gg, expect) in g["mem"]:
        assert oracle.mem(g["chain"]["W"], g["chain"]["a"], k, l, gg) == expect


# ------------------------------------------------------------------ (+) vs 1F1B* grouping
def _greedy_groups(items, T):
    """P:103 verbatim: from the last item backwards, add while the sum stays <= T."""
    n = len(items)
    grp = [0] * n
    g, acc = 1, 0.0
    for i in range(n - 1, -1, -1):
        if acc + items[i] <= T:
            acc += items[i]
        else:
            g += 1
            acc = items[i]
        grp[i] = g
    return grp


def test_oplus_reproduces_greedy_grouping():
    """[S1]: walking items from the end with V <- V (+) u and g = ceil((V+u)/T)
     reproduces the 1F1B* groups of P:103.  Integer items make sums exact."""
    rng = np.random.default_rng(11)
    for _ in range(3000):
        T = float(rng.integers(3, 20))
        items = [float(x) for x in rng.integers(1, int(T) + 1, size=int(rng.integers(1, 12)))]
        grp = _greedy_groups(items, T)
        V = 0.0
        for i in range(len(items) - 1, -1, -1):
            assert math.ceil((V + items[i]) / T) == grp[i]
            V = oracle.oplus(V, items[i], T)


def test_oplus_cases():
    """P:177 on hand values."""
    assert oracle.oplus(0.0, 3.0, 10.0) == 3.0                 # first group
    assert oracle.oplus(4.0, 5.0, 10.0) == 9.0                 # stays in group 1
    assert oracle.oplus(4.0, 6.0, 10.0) == 10.0                # exactly fills group 1
    assert oracle.oplus(4.0, 7.0, 10.0) == 17.0                # new group: 10*1 + 7
    assert oracle.oplus(12.0, 9.0, 10.0) == 29.0               # 20 + 9
    assert oracle.oplus(5.0, 0.0, 10.0) == 5.0                 # zero comm keeps V


def test_g_invariant_under_oplus():
    """[S2]: ceil((V+U)/T) == ceil((V (+) U)/T) whenever U <= T."""
    rng = np.random.default_rng(12)
    for _ in range(20000):
        T = float(rng.uniform(0.5, 5.0))
        V = float(rng.uniform(0.0, 20.0))
        U = float(rng.uniform(0.0, T))
        assert math.ceil((V + U) / T) == math.ceil(oracle.oplus(V, U, T) / T)


# ------------------------------------------------------------------ hand-worked golden examples
def test_golden_three_layer():
    ex = json.load(open(GOLD))["examples"][0]
    r = oracle.solve(ex["chain"], ex["P"], ex["M"], _beta(ex["beta"]), ex["n_m"], ex["n_v"],
                     ex["n_c"], v_range=ex["v_range"])
    e = ex["expect"]
    assert list(r["tau"]) == e["tau"]
    assert r["cand_index"] == e["cand_index"]
    assert r["period"] == e["period"] and r["special_load"] == e["special_load"]
    assert r["load_period"] == e["load_period"]
    assert [list(s) for s in r["stages"]] == e["stages"]


def test_golden_memory_split():
    ex = json.load(open(GOLD))["examples"][1]
    for case in ex["cases"]:
        A, ARG, _ = oracle.table(ex["chain"], ex["P"], case["M"], _beta(ex["beta"]), ex["n_m"],
                                 ex["n_v"], ex["v_range"], ex["tau"])
        root = A[-1, ex["P"] - 1, 0, 0]
        assert root == (INF if case["root"] == "inf" else case["root"])
        if "stages" in case:
            # decision at the root: stage 2..2 on the special processor (2k+o = 5)
            assert ARG[-1, ex["P"] - 1, 0, 0] == 5


# ------------------------------------------------------------------ brute force (O11)
def _rand_case(rng, L=None, P=None):
    L = int(rng.integers(2, 7)) if L is None else L
    P = int(rng.integers(1, 4)) if P is None else P
    ch = chaingen.tiny(rng, L)
    n_m = int(rng.choice([2, 4, 8]))
    n_v = int(rng.choice([4, 8, 16]))
    v_range = int(rng.integers(0, 2))
    total_mem = 3 * int(np.sum(ch["W"])) + 3 * int(np.sum(ch["a"]))
    M = int(total_mem * rng.uniform(0.15, 0.9)) + 1
    beta = float(rng.choice([math.inf, rng.uniform(5.0, 60.0)]))
    return ch, P, M, beta, n_m, n_v, v_range


def test_root_equals_bruteforce_bit_exact():
    """[S3]: the DP root equals the minimum over ALL allocations, evaluated with the
    same grids and rounding, bit for bit (including +inf)."""
    rng = np.random.default_rng(21)
    n_fin = 0
    for _ in range(140):
        ch, P, M, beta, n_m, n_v, vr = _rand_case(rng)
        pre = oracle.prep(ch, P, beta)
        for frac in (0.0, 0.15, 0.35, 0.6, 1.0):
            tau = pre["lb"] + frac * (pre["ub"] - pre["lb"])
            A, ARG, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau)
            bf, _ = bruteforce.root(ch, P, M, beta, n_m, n_v, vr, tau)
            dp = A[-1, P - 1, 0, 0]
            assert dp == bf, (ch, P, M, beta, n_m, n_v, vr, tau, dp, bf)
            n_fin += dp < INF
    assert n_fin > 100     # the fuzz must exercise feasible cases


def test_every_cell_equals_bruteforce():
    """Every cell A[l][p][v][m] (not just the root) equals the brute-force minimum
    over allocations of layers 1..l from state (p, v, m)."""
    rng = np.random.default_rng(22)
    for _ in range(12):
        ch, P, M, beta, n_m, n_v, vr = _rand_case(rng, L=int(rng.integers(2, 5)),
                                                   P=int(rng.integers(1, 4)))
        n_v = 4
        n_m = int(rng.choice([2, 4]))
        pre = oracle.prep(ch, P, beta)
        tau = pre["lb"] + 0.4 * (pre["ub"] - pre["lb"])
        A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau)
        L = len(ch["uF"])
        for l in range(L + 1):
            for p in range(P):
                for v in range(n_v):
                    for m in range(n_m):
                        bf = bruteforce.cell(ch, P, M, beta, n_m, n_v, vr, tau, l, p, v, m)
                        assert A[l, p, v, m] == bf, (l, p, v, m)


def test_traceback_is_an_optimum_and_verified():
    """[S4]: the traced-back allocation's own value equals the root (same summation
    order), and the 1F1B* simulator verifies loads, groups and memory."""
    rng = np.random.default_rng(23)
    checked = 0
    for _ in range(80):
        ch, P, M, beta, n_m, n_v, vr = _rand_case(rng, L=int(rng.integers(3, 8)))
        r = oracle.solve(ch, P, M, beta, n_m, n_v, n_c=12, v_range=vr)
        if r["rc"] != 0:
            assert r["rc"] == oracle.INFEASIBLE
            continue
        val = bruteforce.value_of_stages(ch, P, M, beta, n_m, n_v, vr, r["period"], r["stages"])
        assert val == r["special_load"] == r["root"][r["cand_index"]]
        assert r["load_period"] <= r["period"]
        rep = simulator.check_allocation(ch, P, M, beta, r["period"], r["stages"],
                                         r["load_period"], r["special_load"])
        assert rep["errors"] == [], rep["errors"]
        # no smaller candidate is feasible (O7)
        assert all(not (r["root"][j] <= r["tau"][j]) for j in range(r["cand_index"]))
        checked += 1
    assert checked > 40


def test_continuous_bruteforce_one_sided():
    """O12: the grids round V and m up (Q6), so whatever the discrete DP accepts is
    feasible with exact V and exact memory, with a special load at least as small."""
    rng = np.random.default_rng(24)
    for _ in range(80):
        ch, P, M, beta, n_m, n_v, vr = _rand_case(rng, L=int(rng.integers(2, 6)))
        pre = oracle.prep(ch, P, beta)
        tau = pre["lb"] + rng.uniform(0.05, 0.8) * (pre["ub"] - pre["lb"])
        A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau, with_arg=False)
        dp = A[-1, P - 1, 0, 0]
        cont, _ = bruteforce.root(ch, P, M, beta, n_m, n_v, vr, tau, discrete=False)
        if dp < INF:
            assert cont <= dp


# ------------------------------------------------------------------ special cases (O13)
def test_p1_closed_form():
    """P = 1: feasible iff U(1,L) <= tau and M(1,L,g-1) <= M."""
    rng = np.random.default_rng(31)
    agree = 0
    for _ in range(200):
        L = int(rng.integers(1, 10))
        ch = chaingen.tiny(rng, L)
        pre = oracle.prep(ch, 1, 20.0)
        tau = pre["Up"][-1] * rng.uniform(0.5, 2.0)
        M = int(rng.integers(10, 400))
        A, _, _ = oracle.table(ch, 1, M, 20.0, 8, 8, oracle.PAPER, tau, with_arg=False)
        assert (A[-1, 0, 0, 0] <= tau) == special.p1_feasible(ch, M, tau)
        agree += 1
    assert agree == 200


def test_memory_free_equals_max_coverage():
    """M irrelevant (W = a = 0, so C = 0), SAFE V range: the DP root equals the
    minimum uncovered load of an independent interval-cover DP (integer loads,
    exact sums); under the PAPER range the DP may only be more pessimistic (Q8)."""
    rng = np.random.default_rng(32)
    n_eq = 0
    for _ in range(250):
        L = int(rng.integers(1, 14))
        P = int(rng.integers(1, 6))
        ch = chaingen.tiny(rng, L, integer_times=True, zero_mem=True)
        loads = [int(x + y) for x, y in zip(ch["uF"], ch["uB"])]
        tau = float(rng.integers(max(loads), sum(loads) + 1))
        mc = special.max_coverage(loads, P - 1, tau)
        expect = float(mc) if mc <= tau else INF
        A, _, _ = oracle.table(ch, P, 1, math.inf, 2, 4, oracle.SAFE, tau, with_arg=False)
        assert A[-1, P - 1, 0, 0] == expect, (loads, P, tau)
        A2, _, _ = oracle.table(ch, P, 1, math.inf, 2, 4, oracle.PAPER, tau, with_arg=False)
        assert A2[-1, P - 1, 0, 0] >= expect
        n_eq += expect < INF
    assert n_eq > 100


def test_uniform_chain_threshold():
    """Uniform memory-free chain (SAFE range): the sweep returns the first candidate
    >= ceil(L/P) * u, the textbook optimum."""
    for L, P, u in [(7, 3, 2.0), (12, 4, 1.0), (10, 3, 3.0), (9, 9, 1.0), (5, 1, 2.0), (16, 5, 1.0)]:
        ch = chaingen.uniform(L, u)
        thr = special.uniform_threshold(L, P, u)
        r = oracle.solve(ch, P, 1, math.inf, 2, 8, n_c=64, v_range=oracle.SAFE)
        tau = r["tau"]
        expect_j = min(j for j in range(64) if tau[j] >= thr)
        assert r["cand_index"] == expect_j, (L, P, u)
        assert r["special_load"] <= tau[expect_j]


def test_beta_infinite_means_no_comm():
    ch = chaingen.toy()
    pre = oracle.prep(ch, 2, math.inf)
    assert all(c == 0.0 for c in pre["C"]) and pre["SC"] == 0.0


# ------------------------------------------------------------------ monotonicity (soft)
def test_feasibility_monotone_in_tau_soft():
    """feasibility is non-decreasing in tau.  Discretisation may break it
    in rare cases (the grid moves with tau), so breaks are counted, not failed,
    unless they become common."""
    rng = np.random.default_rng(41)
    breaks = total = 0
    for _ in range(30):
        ch = chaingen.tiny(rng, int(rng.integers(6, 12)))
        P = int(rng.integers(2, 5))
        M = int((3 * ch["W"].sum() + 4 * ch["a"].sum()) * rng.uniform(0.2, 0.6))
        r = oracle.solve(ch, P, M, 30.0, 8, 16, n_c=24, v_range=oracle.PAPER)
        feas = [r["root"][j] <= r["tau"][j] for j in range(24)]
        for j in range(1, 24):
            total += 1
            breaks += feas[j - 1] and not feas[j]
    assert breaks <= 0.05 * total


def test_early_exit_same_winner():
    rng = np.random.default_rng(42)
    for _ in range(20):
        ch, P, M, beta, n_m, n_v, vr = _rand_case(rng, L=8, P=3)
        full = oracle.solve(ch, P, M, beta, n_m, n_v, 20, v_range=vr)
        ee = oracle.solve(ch, P, M, beta, n_m, n_v, 20, v_range=vr, early_exit=True)
        assert full["cand_index"] == ee["cand_index"]
        assert full["stages"] == ee["stages"]
        assert ee["cell_updates"] <= full["cell_updates"]


def test_tie_break_smallest_split_first():
    """Q11: among all (k, N/S) options achieving a cell's minimum, the recorded
    decision is the smallest code 2k+o (smallest split first, N before S) -- a
    rule on the set of optimal options, checked independently of loop order."""
    rng = np.random.default_rng(51)
    n_ties = 0
    for _ in range(25):
        L, P = int(rng.integers(3, 7)), int(rng.integers(2, 4))
        ch = chaingen.tiny(rng, L, integer_times=True, zero_mem=bool(rng.integers(0, 2)))
        M, beta, n_m, n_v, vr = 10**9, math.inf, 2, 4, oracle.SAFE
        pre = oracle.prep(ch, P, beta)
        tau = float(math.ceil(pre["lb"] + 0.3 * (pre["ub"] - pre["lb"])))
        A, ARG, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau)
        for l in range(1, L + 1):
            for p in range(1, P):
                for v in range(n_v):
                    for m in range(n_m):
                        opts = []
                        for k in range(1, l + 1):
                            if pre["Up"][l] - pre["Up"][k - 1] > tau:
                                continue
                            g, nf, d, vn = oracle.transition(ch, P, M, beta, n_m, n_v, vr, tau, k, l, v)
                            if k > 1 and (vn < 0 or pre["C"][k - 1] > tau):
                                continue
                            if nf:
                                opts.append((A[k - 1, p - 1, vn, m], 2 * k))
                            if m + d <= n_m - 1:
                                c = (pre["Up"][l] - pre["Up"][k - 1]) + A[k - 1, p, vn, m + d]
                                if c <= tau:
                                    opts.append((c, 2 * k + 1))
                        best = min([o[0] for o in opts], default=INF)
                        assert A[l, p, v, m] == best
                        codes = [o[1] for o in opts if o[0] == best and best < INF]
                        assert ARG[l, p, v, m] == (min(codes) if codes else -1)
                        n_ties += len(codes) > 1
    assert n_ties > 50


def test_table_monotone_in_processors():
    """Invariant (used by the kernels' sub-row trimming): with one more
    normal GPU available every allocation stays possible (a GPU may stay unused,
    T(0,p,..) = t_P for any p), so A[l][p] <= A[l][p-1] elementwise, and the
    finite cells of a row (l, v) form an up-set {p >= p_first}."""
    rng = np.random.default_rng(71)
    for _ in range(40):
        ch, P, M, beta, n_m, n_v, vr = _rand_case(rng, L=int(rng.integers(3, 10)), P=int(rng.integers(2, 7)))
        pre = oracle.prep(ch, P, beta)
        tau = pre["lb"] + rng.uniform(0.0, 1.0) * (pre["ub"] - pre["lb"])
        A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau, with_arg=False)
        assert np.all(A[:, 1:] <= A[:, :-1])
        fin = np.isfinite(A).any(axis=3)                       # [l][p][v]
        for l in range(A.shape[0]):
            for v in range(n_v):
                col = fin[l, :, v]
                if col.any():
                    first = int(np.argmax(col))
                    assert col[first:].all()


# ------------------------------------------------------------------ communication-bound chains
def _rand_comm_case(rng, L=None, P=None):
    """A family where boundaries are expensive: activations up to 400 bytes with
    beta in [5, 30] (C(i) = 2 a_i / beta up to 160 s against stage loads of a few
    seconds), so C(k-1) > tau prunes splits and a link is often the
    bottleneck of the allocation period."""
    L = int(rng.integers(2, 7)) if L is None else L
    P = int(rng.integers(1, 4)) if P is None else P
    ch = chaingen.tiny(rng, L, a_hi=400)
    n_m = int(rng.choice([2, 4, 8]))
    n_v = int(rng.choice([4, 8, 16]))
    v_range = int(rng.integers(0, 2))
    total_mem = 3 * int(np.sum(ch["W"])) + 3 * int(np.sum(ch["a"]))
    M = int(total_mem * rng.uniform(0.15, 0.9)) + 1
    beta = float(rng.uniform(5.0, 30.0))
    return ch, P, M, beta, n_m, n_v, v_range


def _comm_taus(pre):
    """Periods around the loads, where the comm constraint bites: lb, 1.5 lb, 2.5 lb,
    a tenth of the way to ub, and U(1,L)."""
    lb, ub = pre["lb"], pre["ub"]
    return (lb, 1.5 * lb, 2.5 * lb, lb + 0.1 * (ub - lb), pre["Up"][-1])


def test_root_equals_bruteforce_comm_heavy():
    """[S3] on the communication-bound family: the DP root equals the brute-force
    minimum bit for bit, and the family really exercises C(k-1) > tau."""
    rng = np.random.default_rng(25)
    total = with_c = n_fin = 0
    for _ in range(150):
        ch, P, M, beta, n_m, n_v, vr = _rand_comm_case(rng)
        pre = oracle.prep(ch, P, beta)
        L = len(ch["uF"])
        cmax = max(pre["C"][1:L])
        for tau in _comm_taus(pre):
            A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau, with_arg=False)
            bf, _ = bruteforce.root(ch, P, M, beta, n_m, n_v, vr, tau)
            dp = A[-1, P - 1, 0, 0]
            assert dp == bf, (ch, P, M, beta, n_m, n_v, vr, tau, dp, bf)
            total += 1
            with_c += cmax > tau
            n_fin += dp < INF
    assert with_c >= 0.3 * total and n_fin >= 0.3 * total, (with_c, n_fin, total)


def test_comm_constraint_binds():
    """The C(k-1) <= tau rule changes the answer on this family: with the links made
    free (beta = inf) the same chains are feasible at strictly more of these periods,
    so a DP that ignored the rule would disagree with the brute force above."""
    rng = np.random.default_rng(26)
    differ = 0
    for _ in range(100):
        ch, P, M, beta, n_m, n_v, vr = _rand_comm_case(rng)
        pre = oracle.prep(ch, P, beta)
        for tau in _comm_taus(pre):
            A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau, with_arg=False)
            bf_free, _ = bruteforce.root(ch, P, M, math.inf, n_m, n_v, vr, tau)
            differ += (A[-1, P - 1, 0, 0] == INF) and bf_free < INF
    assert differ >= 20, differ


def test_every_cell_equals_bruteforce_comm_heavy():
    rng = np.random.default_rng(27)
    for _ in range(16):
        ch, P, M, beta, n_m, n_v, vr = _rand_comm_case(rng, L=int(rng.integers(2, 5)),
                                                        P=int(rng.integers(1, 4)))
        n_v = 4
        n_m = int(rng.choice([2, 4]))
        pre = oracle.prep(ch, P, beta)
        tau = 1.5 * pre["lb"]
        A, _, _ = oracle.table(ch, P, M, beta, n_m, n_v, vr, tau)
        L = len(ch["uF"])
        for l in range(L + 1):
            for p in range(P):
                for v in range(n_v):
                    for m in range(n_m):
                        bf = bruteforce.cell(ch, P, M, beta, n_m, n_v, vr, tau, l, p, v, m)
                        assert A[l, p, v, m] == bf, (l, p, v, m)


def test_traceback_verified_comm_heavy():
    """[S4] on the communication-bound family, with a grid that starts near lb: the
    simulator recomputes the allocation period including every link, so a
    load_period that missed the link term, or an allocation with a link above tau,
    fails here."""
    rng = np.random.default_rng(28)
    checked = link_bound = 0
    for _ in range(200):
        ch, P, M, beta, n_m, n_v, vr = _rand_comm_case(rng, L=int(rng.integers(3, 8)))
        r = oracle.solve(ch, P, M, beta, n_m, n_v, n_c=400, v_range=vr)
        if r["rc"] != 0:
            continue
        val = bruteforce.value_of_stages(ch, P, M, beta, n_m, n_v, vr, r["period"], r["stages"])
        assert val == r["special_load"] == r["root"][r["cand_index"]]
        rep = simulator.check_allocation(ch, P, M, beta, r["period"], r["stages"],
                                         r["load_period"], r["special_load"], build_pattern=False)
        assert rep["errors"] == [], rep["errors"]
        loads = [sum(ch["uF"][i] + ch["uB"][i] for i in range(k - 1, l)) for (k, l, p) in r["stages"]
                 if p != P - 1]
        links = [2.0 * ch["a"][k - 1] / beta for (k, l, p) in r["stages"] if k > 1]
        link_bound += bool(links) and max(links) > max(loads + [r["special_load"]])
        checked += 1
    assert checked > 100 and link_bound >= 10, (checked, link_bound)


def test_golden_communication_forces_merge():
    ex = json.load(open(GOLD))["examples"][2]
    r = oracle.solve(ex["chain"], ex["P"], ex["M"], _beta(ex["beta"]), ex["n_m"], ex["n_v"],
                     ex["n_c"], v_range=ex["v_range"])
    e = ex["expect"]
    assert list(r["tau"][:3]) == e["tau_first"]
    assert r["root"][0] == INF
    assert r["cand_index"] == e["cand_index"]
    assert r["period"] == e["period"] and r["special_load"] == e["special_load"]
    assert r["load_period"] == e["load_period"]
    assert [list(s) for s in r["stages"]] == e["stages"]


def test_golden_tau_grid_rounding():
    ex = json.load(open(GOLD))["examples"][4]
    r = oracle.solve(ex["chain"], ex["P"], ex["M"], _beta(ex["beta"]), ex["n_m"], ex["n_v"],
                     ex["n_c"], v_range=ex["v_range"])
    assert [float.fromhex(h) for h in ex["expect"]["tau_hex"]] == list(r["tau"])
