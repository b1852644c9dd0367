"""O10: 1F1B* simulator and allocation checker.  TEST INFRASTRUCTURE ONLY.

Given an allocation returned by MadPipe-DP (stages (first, last, proc); normal
processors 0..P-2, special processor P-1) and its period tau, this module
re-derives, independently of both the C oracle and the CUDA library:

1. the resource loads, by left-to-right per-stage sums of u_F + u_B (a
   different summation order from the prefix differences U(k,l) of P:155),
   and the allocation period = load of the most loaded resource, GPU or
   communication link (reading Q17);
2. the 1F1B* groups WITHOUT discretisation: stages and their boundary
   communications (each a "layer" of duration C(l) = 2 a_l / beta)
   walked from the end with the exact (+) of P:177, giving each stage's
   group index g_s;
3. the memory checks: M(k,l,g_s) <= M on every normal GPU (exact by P:113 and
   Proposition 1), and sum over special stages of M(k,l,g_s - 1) <= M (the
   DP's model of the special processor);
4. the special processor's Figure 5 memory peaks (worst: sum g_i abar_i; best:
   max_i g_i abar_i + sum_{j!=i} (g_j - 1) abar_j, with abar_s = sum_{i in s}
   a_{i-1} from P:217), reported, not asserted (reading Q20);
5. for allocations whose special processor holds <= 1 stage (a contiguous
   allocation), the 1F1B* periodic pattern itself on the 2N-1 transformed
   chain: start times and index shifts of every forward and
   backward operation, a check of every dependency of Figure 1 across periods
    and of the number of active batches per stage, which must be
   exactly its group index (Proposition 1).
"""
from __future__ import annotations

import math


def _stage_loads(ch, stages):
    uF, uB = ch["uF"], ch["uB"]
    loads, fw, bw = [], [], []
    for (k, l, _p) in stages:
        s, f, b = 0.0, 0.0, 0.0
        for i in range(k, l + 1):
            s += float(uF[i - 1]) + float(uB[i - 1])
            f += float(uF[i - 1])
            b += float(uB[i - 1])
        loads.append(s); fw.append(f); bw.append(b)
    return loads, fw, bw


def _oplus(x, y, tau):
    cx = math.ceil(x / tau)
    if cx == math.ceil((x + y) / tau):
        return x + y
    return tau * cx + y


def _mem(ch, k, l, g):
    W, a, L = ch["W"], ch["a"], len(ch["uF"])
    m = 0
    for i in range(k, l + 1):
        m += 3 * int(W[i - 1]) + g * int(a[i - 1])
    if k > 1:
        m += 2 * int(a[k - 1])
    if l < L:
        m += 2 * int(a[l])
    return m


def exact_groups(ch, stages, tau, beta):
    """Group index of every stage with exact delays (P:103 via the (+) of P:177)."""
    a = ch["a"]
    loads, _, _ = _stage_loads(ch, stages)
    g = [0] * len(stages)
    V = 0.0
    for s in range(len(stages) - 1, -1, -1):
        k = stages[s][0]
        g[s] = math.ceil((V + loads[s]) / tau)
        c = (2.0 * float(a[k - 1])) / beta if k > 1 else 0.0
        V = _oplus(_oplus(V, loads[s], tau), c, tau)
    return g


def check_allocation(ch, P, M, beta, tau, stages, load_period=None, special_load=None,
                     rel_tol=1e-12, build_pattern=True):
    """Run checks 1-5 on an allocation; returns a report dict.  Hard failures are
    collected in report["errors"] (empty list = allocation verified)."""
    L = len(ch["uF"])
    a = ch["a"]
    errors = []
    # -- structure: stages tile 1..L in order
    pos = 1
    for (k, l, p) in stages:
        if k != pos or l < k or not (0 <= p <= P - 1):
            errors.append("stages do not tile the chain: %r" % (stages,))
            break
        pos = l + 1
    if pos != L + 1:
        errors.append("stages do not cover layers 1..L")
    normals = [p for (_, _, p) in stages if p != P - 1]
    if len(set(normals)) != len(normals) or len(normals) > P - 1:
        errors.append("a normal processor holds more than one stage")
    # -- 1. loads
    loads, fw, bw = _stage_loads(ch, stages)
    special = 0.0
    lp = 0.0
    for s, (k, l, p) in enumerate(stages):
        if p == P - 1:
            special += loads[s]
        else:
            lp = max(lp, loads[s])
        if k > 1:
            lp = max(lp, (2.0 * float(a[k - 1])) / beta)
    lp = max(lp, special)
    if load_period is not None and abs(lp - load_period) > rel_tol * max(load_period, 1e-300):
        errors.append("load_period %r vs simulated %r" % (load_period, lp))
    if special_load is not None and abs(special - special_load) > rel_tol * max(special_load, 1e-300):
        errors.append("special_load %r vs simulated %r" % (special_load, special))
    if lp > tau * (1.0 + rel_tol):
        errors.append("allocation period %r exceeds tau %r" % (lp, tau))
    # -- 2./3. exact groups and memory
    g = exact_groups(ch, stages, tau, beta)
    normal_mem = []
    special_mem = 0
    abar = []
    for s, (k, l, p) in enumerate(stages):
        abar.append(sum(int(a[i - 1]) for i in range(k, l + 1)))
        if p == P - 1:
            special_mem += _mem(ch, k, l, g[s] - 1)
        else:
            mm = _mem(ch, k, l, g[s])
            normal_mem.append(mm)
            if mm > M:
                errors.append("normal stage %r needs %d > M=%d" % (stages[s], mm, M))
    if special_mem > M:
        errors.append("special processor model memory %d > M=%d" % (special_mem, M))
    # -- 4. Figure 5 peaks on the special processor
    sp = [s for s, (_, _, p) in enumerate(stages) if p == P - 1]
    fixed = sum(_mem(ch, stages[s][0], stages[s][1], 0) for s in sp)
    worst = fixed + sum(g[s] * abar[s] for s in sp)
    best = fixed + (max(g[i] * abar[i] + sum((g[j] - 1) * abar[j] for j in sp if j != i) for i in sp)
                    if sp else 0)
    report = dict(errors=errors, load_period=lp, special_load=special, groups=g,
                  normal_mem=normal_mem, special_mem_model=special_mem,
                  special_peak_worst=worst, special_peak_best=best,
                  needs_ilp=bool(sp) and best > M, pattern=None)
    # -- 5. 1F1B* pattern for contiguous allocations
    if build_pattern and len(sp) <= 1 and not errors:
        report["pattern"] = one_f_one_b_star(ch, stages, tau, beta, g, errors)
    return report


def one_f_one_b_star(ch, stages, tau, beta, g_expected, errors):
    """Build the 1F1B* pattern on the transformed chain of stages and
    communications, then verify it over several periods."""
    a = ch["a"]
    _, fw, bw = _stage_loads(ch, stages)
    # transformed chain: items alternate stage, comm, stage, ... (2N-1 items)
    items = []      # (kind, index, uF, uB)
    for s, (k, l, _p) in enumerate(stages):
        if s > 0:
            c = float(a[k - 1]) / beta        # a^(k-1) forward, b^(k-1) backward
            items.append(("comm", s, c, c))
        items.append(("stage", s, fw[s], bw[s]))
    n = len(items)
    U = [it[2] + it[3] for it in items]
    # phase 1: groups from the last item backwards while sum U <= T
    group = [0] * n
    gi, acc, i = 1, 0.0, n - 1
    while i >= 0:
        if acc + U[i] <= tau or acc == 0.0:
            acc += U[i]
            group[i] = gi
            i -= 1
        else:
            gi += 1
            acc = 0.0
    # stage group indices must equal the exact-(+) ones (identity [S1])
    for j, it in enumerate(items):
        if it[0] == "stage" and group[j] != g_expected[it[1]]:
            errors.append("1F1B* group of stage %d is %d, (+) walk gave %d"
                          % (it[1], group[j], g_expected[it[1]]))
    # phase 2: forward ops chained with shift 0; each group's backward ops
    # right after its last forward op, in reverse, with shift g-1; then wrap mod T.
    tF, tB = [0.0] * n, [0.0] * n
    hF, hB = [0] * n, [0] * n
    t = 0.0
    for j in range(n):
        tF[j] = t
        t += items[j][2]
    j = n - 1
    while j >= 0:
        gg = group[j]
        first = j
        while first - 1 >= 0 and group[first - 1] == gg:
            first -= 1
        tb = tF[j] + items[j][2]
        for q in range(j, first - 1, -1):
            tB[q] = tb
            hB[q] = gg - 1
            tb += items[q][3]
        j = first - 1
    # unwrapped absolute schedule of batch b: op starts at (b + h) T + t
    # dependency checks for batch 0 with the unwrapped (t, h) (wrapping is a
    # relabelling that preserves (b + h) T + t):
    eps = 1e-9 * tau

    def start_F(j, b=0):
        return (b + hF[j]) * tau + tF[j]

    def start_B(j, b=0):
        return (b + hB[j]) * tau + tB[j]

    for j in range(n - 1):
        if start_F(j + 1) + eps < start_F(j) + items[j][2]:
            errors.append("F dependency violated at item %d" % j)
        if start_B(j) + eps < start_B(j + 1) + items[j + 1][3]:
            errors.append("B dependency violated at item %d" % j)
    if start_B(n - 1) + eps < start_F(n - 1) + items[n - 1][2]:
        errors.append("F_L -> B_L dependency violated")
    # resource constraint: F and B of one item must not overlap modulo T
    for j in range(n):
        f0 = tF[j] % tau
        b0 = tB[j] % tau
        if U[j] > tau * (1 + 1e-12):
            errors.append("item %d load exceeds the period" % j)
            continue
        d = (b0 - f0) % tau
        if d + eps < items[j][2] or (tau - d) + eps < items[j][3]:
            errors.append("F/B of item %d overlap within a period" % j)
    # wrap into [0, T): start lowered by T, shift increased by 1
    pattern = []
    for j in range(n):
        ft, fh = tF[j], hF[j]
        while ft >= tau:
            ft -= tau; fh += 1
        bt, bh = tB[j], hB[j]
        while bt >= tau:
            bt -= tau; bh += 1
        pattern.append(dict(kind=items[j][0], index=items[j][1], F=(ft, fh), B=(bt, bh)))
    # active batches: max_t #F started - #B started = ceil(lifetime / T)
    active = []
    for j in range(n):
        life = (hB[j] - hF[j]) * tau + (tB[j] - tF[j])
        act = math.ceil(life / tau - 1e-12)
        active.append(act)
        if items[j][0] == "stage" and act != group[j]:
            errors.append("stage %d keeps %d active batches, group index %d"
                          % (items[j][1], act, group[j]))
    return dict(items=[(it[0], it[1]) for it in items], group=group, active=active,
                pattern=pattern)
