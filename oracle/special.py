"""O13: special-case solvers used as independent pins.  TEST INFRASTRUCTURE ONLY.

* `p1_feasible`     -- P = 1: all layers on the special processor; feasible iff
                       U(1,L) <= tau and M(1,L,g-1) <= M (P:193 with p = 0).
* `max_coverage`    -- memory-free chains (W = a = 0, hence C = 0): a normal
                       processor can take any stage with load <= tau, the
                       special processor takes everything else.  MadPipe-DP in
                       decision form then asks for at most P-1 disjoint
                       intervals, each of load <= tau, whose complement has load
                       <= tau; its root value is the smallest such complement.
                       Computed here by a textbook interval-cover DP that
                       maximises the covered load (integer times, so every sum
                       is exact).
* `uniform_threshold` -- uniform memory-free chain of L layers of load u on P
                       processors: the optimal period is ceil(L/P) * u.
"""
from __future__ import annotations

import math


def p1_feasible(ch, M, tau):
    uF, uB, W, a = ch["uF"], ch["uB"], ch["W"], ch["a"]
    L = len(uF)
    total = 0.0
    for i in range(L):
        total = total + (float(uF[i]) + float(uB[i]))
    if total > tau:
        return False
    g = math.ceil(total / tau)
    # M(1, L, g-1): no communication buffers at k=1 and l=L
    mem = sum(3 * int(W[i]) + (g - 1) * int(a[i]) for i in range(L))
    return mem <= M


def max_coverage(loads, n_intervals, tau):
    """Min uncovered load when covering with <= n_intervals disjoint contiguous
    intervals of load <= tau each.  `loads` are exact (integers)."""
    L = len(loads)
    NEG = -1
    # best[l][q] = max covered load of layers 1..l using <= q intervals
    best = [[0] * (n_intervals + 1) for _ in range(L + 1)]
    for l in range(1, L + 1):
        for q in range(n_intervals + 1):
            b = best[l - 1][q]                   # layer l uncovered
            if q > 0:
                s = 0
                for k in range(l, 0, -1):        # interval k..l
                    s += loads[k - 1]
                    if s > tau:
                        break
                    cand = best[k - 1][q - 1] + s
                    if cand > b:
                        b = cand
            best[l][q] = b
    total = sum(loads)
    del NEG
    return total - best[L][n_intervals]


def uniform_threshold(L, P, u):
    return math.ceil(L / P) * u
