"""O11 / O12: exhaustive enumeration of allocations on tiny chains.
TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Independent of madpipe_oracle.c: it re-derives every step from the paper, but
instead of a recursion over (l, p, v, m) it enumerates every partitioning of
layers 1..l into stages and every N/S assignment (section 4.2), then
evaluates each allocation by walking it from the end exactly as MadPipe-DP's
decisions would:

* a stage (k..l) on a normal processor needs U(k,l) <= tau and
  M(k,l,g(k,l,V)) <= M; it uses one of the p normal processors;
* a stage on the special processor adds U(k,l) to its load and
  M(k,l,g-1) to its memory;
* every boundary k-1 (k>1) needs C(k-1) <= tau (reading Q2);
* the delay for the stage on the left is V' = (V (+) U(k,l)) (+) C(k-1)
  (P:179 with reading Q2);
* when no normal processor is left, the whole remaining prefix 1..l is one
  stage on the special processor (reading Q10).

`discrete=True` (O11) applies the DP's grids and rounding (readings Q6-Q8):
V is rounded up to the next multiple of dV (overflow past the range is
infeasible under the PAPER preset, saturates under SAFE), the special memory
is counted in levels of M/(n_m-1), rounded up per stage.  The special load is
accumulated from the chain start as  acc = U(k,l) + acc  (reading Q13), so the
minimum over allocations must equal the DP root bit for bit.

`discrete=False` (O12) uses exact V and exact memory (no grids): a one-sided
bound -- every allocation the discrete DP accepts is accepted here.
"""
from __future__ import annotations

import math

INF = math.inf


class Chain:
    """Prefix sums written out from P:155 and P:159 (own copy, no shared code)."""

    def __init__(self, ch, P, M, beta, n_m, n_v, v_range):
        self.uF = [float(x) for x in ch["uF"]]
        self.uB = [float(x) for x in ch["uB"]]
        self.W = [int(x) for x in ch["W"]]
        self.a = [int(x) for x in ch["a"]]
        self.L = len(self.uF)
        self.P, self.M, self.beta = P, int(M), float(beta)
        self.n_m, self.n_v, self.v_range = n_m, n_v, v_range
        L = self.L
        self.Up = [0.0] * (L + 1)
        for i in range(1, L + 1):
            self.Up[i] = self.Up[i - 1] + (self.uF[i - 1] + self.uB[i - 1])
        self.C = [0.0] * (L + 1)
        self.SC = 0.0
        for i in range(1, L):
            self.C[i] = (2.0 * float(self.a[i])) / self.beta
            self.SC = self.SC + self.C[i]

    def U(self, k, l):
        return self.Up[l] - self.Up[k - 1]

    def mem(self, k, l, g):
        # sum_{i=k..l} (3 W_i + g a_{i-1}) + 2 (a_{k-1} + a_l), buffers dropped at k=1, l=L
        m = sum(3 * self.W[i - 1] + g * self.a[i - 1] for i in range(k, l + 1))
        if k > 1:
            m += 2 * self.a[k - 1]
        if l < self.L:
            m += 2 * self.a[l]
        return m

    def vmax(self, tau):
        if self.v_range == 1:
            return 2.0 * (self.Up[self.L] + self.SC) + tau
        return self.Up[self.L] + self.SC


def oplus(x, y, tau):
    cx = math.ceil(x / tau)
    s = x + y
    if cx == math.ceil(s / tau):
        return s
    return tau * cx + y


def partitions(l):
    """All partitions of layers 1..l into contiguous stages, as lists of (k, l)."""
    if l == 0:
        yield []
        return
    for k in range(1, l + 1):
        for rest in partitions(k - 1):
            yield rest + [(k, l)]


def allocations(l, p):
    """All (stage, kind) lists for layers 1..l with p normal processors available,
    following the DP's shape: when p normal processors have been used walking
    from the end, the remaining prefix is one special stage (Q10)."""
    if l == 0:
        yield []
        return
    if p == 0:
        yield [((1, l), 1)]
        return
    for k in range(1, l + 1):
        for o in (0, 1):
            for rest in allocations(k - 1, p - 1 if o == 0 else p):
                yield rest + [((k, l), o)]


def evaluate(c: Chain, tau, alloc, p, v, m, discrete=True):
    """Special load of `alloc` (chain order) of layers 1..l starting from state
    (p normal processors, delay level v, special memory level m), or INF."""
    n_m, M = c.n_m, c.M
    if discrete:
        dV = c.vmax(tau) / float(c.n_v - 1)
        V = float(v) * dV
        used = m                       # levels
    else:
        V = v                          # exact delay
        used = m                       # exact bytes
    specials = []
    for idx in range(len(alloc) - 1, -1, -1):
        (k, l), o = alloc[idx]
        Ukl = c.U(k, l)
        if Ukl > tau:
            return INF
        if k > 1 and c.C[k - 1] > tau:
            return INF
        g = math.ceil((V + Ukl) / tau)
        if o == 0:
            if p == 0 or c.mem(k, l, g) > M:
                return INF
            p -= 1
        else:
            D = c.mem(k, l, g - 1)
            if discrete:
                d = -(-(D * (n_m - 1)) // M)
                if used + d > n_m - 1:
                    return INF
                used += d
            else:
                if used + D > M:
                    return INF
                used += D
            specials.append(Ukl)
        if k > 1:
            Vn = oplus(oplus(V, Ukl, tau), c.C[k - 1], tau)
            if discrete:
                q = math.ceil(Vn / dV)
                if q > c.n_v - 1:
                    if c.v_range == 1:
                        q = c.n_v - 1
                    else:
                        return INF
                V = float(q) * dV
            else:
                V = Vn
    acc = 0.0
    for Ukl in reversed(specials):      # chain order: acc = U(k,l) + acc
        acc = Ukl + acc
    return acc if acc <= tau else INF


def cell(ch, P, M, beta, n_m, n_v, v_range, tau, l, p, v=0, m=0, discrete=True):
    """Brute-force value of DP cell (l, p, v, m): min over allocations of 1..l."""
    c = Chain(ch, P, M, beta, n_m, n_v, v_range)
    if l == 0:
        return 0.0
    best = INF
    for alloc in allocations(l, p):
        val = evaluate(c, tau, alloc, p, v, m, discrete)
        if val < best:
            best = val
    return best


def root(ch, P, M, beta, n_m, n_v, v_range, tau, discrete=True):
    """Brute-force T(L, P-1, 0, 0, 0) in decision form, plus the optimal allocations."""
    c = Chain(ch, P, M, beta, n_m, n_v, v_range)
    best, arg = INF, []
    for alloc in allocations(c.L, P - 1):
        val = evaluate(c, tau, alloc, P - 1, 0.0 if not discrete else 0, 0, discrete)
        if val < best:
            best, arg = val, [alloc]
        elif val == best and val < INF:
            arg.append(alloc)
    return best, arg


def value_of_stages(ch, P, M, beta, n_m, n_v, v_range, tau, stages):
    """Discrete evaluation of an allocation given as [(first, last, proc)]."""
    c = Chain(ch, P, M, beta, n_m, n_v, v_range)
    alloc = [((f, l), 1 if pr == P - 1 else 0) for (f, l, pr) in stages]
    return evaluate(c, tau, alloc, P - 1, 0, 0, True)


# --------------------------------------------------------------------------
# NEXT row f1: the paper-literal optimisation form (t_P discretised)
# --------------------------------------------------------------------------
def literal_evaluate(c: Chain, That, n_t, alloc, p, t, m, v):
    """Period the literal DP assigns to `alloc` (chain order) of layers 1..l from
    state (p, t, m, v): the max of every term met along the path -- normal stage
    loads U(k,l), boundary times C(k-1), the special load t*dt after each special
    stage (each stage's load rounded up to the t grid), U(1,l) + t*dt at the p = 0
    base, t*dt at l = 0.  INF if a constraint fails."""
    n_m, M = c.n_m, c.M
    dV = c.vmax(That) / float(c.n_v - 1)
    dt = c.Up[c.L] / float(n_t - 1)
    V = float(v) * dV
    terms = []
    for idx in range(len(alloc) - 1, -1, -1):
        (k, l), o = alloc[idx]
        Ukl = c.U(k, l)
        g = math.ceil((V + Ukl) / That)
        if p == 0:                                   # base: the single remaining stage 1..l
            D = c.mem(k, l, g - 1)
            if k != 1 or o != 1 or m + -(-(D * (n_m - 1)) // M) > n_m - 1:
                return INF
            terms.append(Ukl + float(t) * dt)
            return max(terms)
        if k > 1:
            terms.append(c.C[k - 1])
        if o == 0:
            if c.mem(k, l, g) > M:
                return INF
            terms.append(Ukl)
            p -= 1
        else:
            D = c.mem(k, l, g - 1)
            dd = -(-(D * (n_m - 1)) // M)
            ts = math.ceil(Ukl / dt)
            if m + dd > n_m - 1 or t + ts > n_t - 1:
                return INF
            m += dd
            t += ts
            terms.append(float(t) * dt)
        if k > 1:
            Vn = oplus(oplus(V, Ukl, That), c.C[k - 1], That)
            q = math.ceil(Vn / dV)
            if q > c.n_v - 1:
                return INF
            V = float(q) * dV
    terms.append(float(t) * dt)                        # T(0, p, t_P, ...) = t_P
    return max(terms)


def literal_root(ch, P, M, beta, n_m, n_v, n_t, That):
    c = Chain(ch, P, M, beta, n_m, n_v, 0)
    best = INF
    for alloc in allocations(c.L, P - 1):
        val = literal_evaluate(c, That, n_t, alloc, P - 1, 0, 0, 0)
        if val < best:
            best = val
    return best
