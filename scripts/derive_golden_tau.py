#!/usr/bin/env python
"""Derive the candidate-grid golden of tests/golden/hand_worked.json ("tau_grid_rounding").

Independent of oracle/ and of the CUDA library: exact rational arithmetic
(fractions.Fraction) plus an explicit IEEE-754 binary64 round-to-nearest-even
written from its definition.  It evaluates the O3 grid formula of reading Q14,

    tau_j = lb + j * ((ub - lb) / (n_c - 1)),   lb = U(1,L)/P,  ub = U(1,L) + sum C

one correctly rounded operation at a time, in that order, and prints every
intermediate as an exact fraction and as a hex float.  Chain: one layer,
uF = 0.25, uB = 0.75 (U(1,1) = 1 exactly), P = 2, beta = inf (sum C = 0),
n_c = 7, so lb = 1/2, ub = 1 and the step 1/12 is not representable.
"""
from fractions import Fraction as F


def rne(x: F) -> F:
    """Round a positive rational to the nearest binary64 value, ties to even."""
    assert x > 0
    e = 0
    while x >= 2 ** (e + 1):
        e += 1
    while x < 2 ** e:
        e -= 1
    ulp = F(2) ** (e - 52)               # 53-bit significand in [2^e, 2^(e+1))
    q, r = divmod(x, ulp)
    q = int(q)
    if r * 2 > ulp or (r * 2 == ulp and q % 2 == 1):
        q += 1
    return q * ulp


def hexf(x: F) -> str:
    return float(x).hex()   # float(x) is exact here: x is already a binary64 value


def main():
    U = rne(F(1, 4) + F(3, 4))           # uF + uB of the single layer
    Up1 = rne(F(0) + U)                  # O1 prefix sum
    lb = rne(Up1 / 2)                    # Alg. 1 line 1: U(1,L)/P
    ub = rne(Up1 + 0)                    # line 2: U(1,L) + sum C, sum C = 0
    n_c = 7
    diff = rne(ub - lb)
    step = rne(diff / (n_c - 1))
    print("lb =", lb, "ub =", ub, "step = fl(1/12) =", step, hexf(step))
    taus = []
    for j in range(n_c):
        prod = rne(j * step) if j else F(0)
        tau = rne(lb + prod)
        taus.append(tau)
        alt = rne(lb + rne(rne(j * diff) / (n_c - 1))) if j else lb
        print("j=%d  j*step=%s  tau=%s (%s)  [reassociated: %s]" % (j, prod, tau, hexf(tau), hexf(alt)))
    print([hexf(t) for t in taus])


if __name__ == "__main__":
    main()
