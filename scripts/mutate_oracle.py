#!/usr/bin/env python
"""Mutation check of the CPU oracle's pins.

Each mutation is one plausible single-line mistake in oracle/madpipe_oracle.c
(a dropped term, a wrong index, a wrong rounding, the garbled printed order of
Algorithm 1, ...).  For each one the script compiles a mutated copy under /tmp,
points the oracle package at it (ORACLE_LIB) and runs the CPU pin suites.  A
mutation is "caught" when at least one pin fails.  The report is written as a
markdown table (default profiles/r02_oracle_mutations.md).

    python scripts/mutate_oracle.py [--out FILE] [--only NAME ...]
"""
from __future__ import annotations

import argparse
import os
import subprocess
import sys
import tempfile
import time
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "madpipe_oracle.c")
PIN_TESTS = ["tests/test_oracle_pins.py", "tests/test_oracle_literal.py", "tests/test_simulator.py"]

# Mutants that cannot change any result (proved in the note), reported as "equivalent"
EQUIVALENT = {
    "literal: S period term t dt instead of t' dt":
        "every literal cell satisfies T(l,p,t,..) >= t dt (base T(0,p,t) = t dt, and each option "
        "takes a max with a cell at t' >= t), so max(t dt, C, T(k-1,p,t',..)) = max(t' dt, C, T(k-1,p,t',..))",
}

# (name, passage the correct line follows, old text, new text)
MUTATIONS = [
    ("drop C(k-1) > tau skip", "P:183/P:187 (C(k-1) <= T in T_N, T_S)",
     "if (k > 1 && (t.vn == VN_OVERFLOW || c->C[k - 1] > tau)) continue;",
     "if (k > 1 && (t.vn == VN_OVERFLOW)) continue;"),
    ("drop link term of load_period", "P:153 (period = max load over GPUs and links)",
     "if (first[i] > 1 && c->C[first[i] - 1] > lp) lp = c->C[first[i] - 1];",
     "(void)0;"),
    ("drop special load from load_period", "P:153, O9",
     "*load_period = root > lp ? root : lp;", "*load_period = lp;"),
    ("Alg.1 printed ub <- min(ub, T)", "P:205, reading Q15",
     "if (Tm < ub) ub = Tm;", "if (T < ub) ub = T;"),
    ("Alg.1 printed lb <- max(lb, That)", "P:205, reading Q15",
     "if (lo > lb) lb = lo;", "if (That > lb) lb = That;"),
    ("Alg.1 best by T instead of max(T, That)", "P:199",
     "if (Tm < best) { best = Tm; bi = i; }", "if (T < best) { best = T; bi = i; }"),
    ("tau grid reassociated", "O3 / reading Q14",
     "return lb + (double)j * ((ub - lb) / (double)(n_c - 1));",
     "return lb + ((double)j * (ub - lb)) / (double)(n_c - 1);"),
    ("lb = U/(P-1)", "P:205 line 1",
     "double lb = c->Up[c->L] / (double)c->P;          /* Alg. 1 line 1 (P:205) */",
     "double lb = c->Up[c->L] / (double)(c->P + 1);"),
    ("C(k) instead of C(k-1) in V'", "P:179 with reading Q2",
     "double Vn = oracle_oplus(oracle_oplus(V, Ukl, tau), c->C[k - 1], tau);",
     "double Vn = oracle_oplus(oracle_oplus(V, Ukl, tau), c->C[k], tau);"),
    ("(+) operands swapped in V'", "P:179",
     "double Vn = oracle_oplus(oracle_oplus(V, Ukl, tau), c->C[k - 1], tau);",
     "double Vn = oracle_oplus(oracle_oplus(V, c->C[k - 1], tau), Ukl, tau);"),
    ("(+) without grouping", "P:177",
     "    return tau * cx + y;\n}", "    return s;\n}"),
    ("a_k instead of a_{k-1} buffer", "P:159",
     "if (k > 1) m += 2 * c->a[k - 1];", "if (k > 1) m += 2 * c->a[k];"),
    ("Ap sums a_i instead of a_{i-1}", "P:159",
     "c->Ap[i] = c->Ap[i - 1] + a[i - 1];", "c->Ap[i] = c->Ap[i - 1] + a[i];"),
    ("sum C over 1..L (Q4 off by one)", "P:205 line 2, reading Q4",
     "    for (int i = 1; i <= L - 1; i++) {\n        c->C[i] = (2.0 * (double)a[i]) / beta;",
     "    for (int i = 1; i <= L; i++) {\n        c->C[i] = (2.0 * (double)a[i]) / beta;"),
    ("N reads row p instead of p-1", "P:183",
     "double cand = A[IDX(c, k - 1, p - 1, t.vn, m)];", "double cand = A[IDX(c, k - 1, p, t.vn, m)];"),
    ("floor for ceil in g", "P:159",
     "t.g = (int64_t)ceil((V + Ukl) / tau);", "t.g = (int64_t)floor((V + Ukl) / tau) + 1;"),
    ("g instead of g-1 for the special GPU", "P:161-163, P:185",
     "int64_t D = Mem(c, k, l, t.g - 1);", "int64_t D = Mem(c, k, l, t.g);"),
    ("g-1 instead of g for a normal GPU", "P:181",
     "t.nf = Mem(c, k, l, t.g) <= c->M;", "t.nf = Mem(c, k, l, t.g - 1) <= c->M;"),
    ("memory shift rounded down", "reading Q6/Q7",
     "t.d = (D * (int64_t)(c->n_m - 1) + c->M - 1) / c->M;", "t.d = (D * (int64_t)(c->n_m - 1)) / c->M;"),
    ("delay level rounded down", "reading Q6",
     "double q = ceil(Vn / dV);", "double q = floor(Vn / dV);"),
    ("PAPER V range without sum C", "P:233, reading Q8",
     "    return c->Up[c->L] + c->SC;\n}", "    return c->Up[c->L];\n}"),
    ("drop the S clamp to tau", "reading Q12",
     "if (cand <= tau && cand < *best)", "if (cand < *best)"),
    ("drop U(1,l) <= tau in the base row", "P:193",
     "int ok = (U1l <= tau) && ((int64_t)m + t.d <= (int64_t)(n_m - 1));",
     "int ok = ((int64_t)m + t.d <= (int64_t)(n_m - 1));"),
    ("tie-break: largest split wins", "reading Q11",
     "if (cand < *best) { *best = cand; if (ARG) ARG[IDX(c, l, p, v, m)] = 2 * k; }",
     "if (cand <= *best) { *best = cand; if (ARG) ARG[IDX(c, l, p, v, m)] = 2 * k; }"),
    ("window: U(k,l) < tau", "O5",
     "if (U(c, k, l) <= tau) return k;", "if (U(c, k, l) < tau) return k;"),
    ("traceback keeps delay level", "P:195",
     "        v = t.vn;\n        l = k - 1;\n    }\n    /* reverse", "        l = k - 1;\n    }\n    /* reverse"),
    ("literal: S period term t dt instead of t' dt", "P:187, reading L1",
     "double cand = dmax(dmax((double)t2 * dt, Ck),", "double cand = dmax(dmax((double)t * dt, Ck),"),
    ("literal: N without C(k-1)", "P:183",
     "double cand = dmax(dmax(Ukl, Ck), A[LIDX(c, n_t, k - 1, p - 1, t, tr.vn, m)]);",
     "double cand = dmax(Ukl, A[LIDX(c, n_t, k - 1, p - 1, t, tr.vn, m)]);"),
    ("literal: t grid step rounded down", "reading L1",
     "int64_t dts = (int64_t)ceil(Ukl / dt);", "int64_t dts = (int64_t)floor(Ukl / dt);"),
]


def _one(i, name, cite, old, new, src, tmp):
    n = src.count(old)
    if n != 1:
        return (name, cite, "PATTERN x%d" % n, "", 0.0)
    cpath = os.path.join(tmp, "m%02d.c" % i)
    lpath = os.path.join(tmp, "m%02d.so" % i)
    open(cpath, "w").write(src.replace(old, new))
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                           "-fPIC", "-shared", "-w", "-o", lpath, cpath, "-lm"])
    env = dict(os.environ, ORACLE_LIB=lpath, OMP_NUM_THREADS="1")
    t0 = time.time()
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "not gpu", *PIN_TESTS],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    failed = ""
    for ln in r.stdout.splitlines():
        if ln.startswith("FAILED"):
            failed = ln.split(" ")[1].split("::")[-1]
            break
    status = "caught" if r.returncode != 0 else ("equivalent" if name in EQUIVALENT else "SURVIVED")
    return (name, cite, status, failed, time.time() - t0)


def run(out, only=None, jobs=None, quiet=False):
    src = open(SRC).read()
    tmp = tempfile.mkdtemp(prefix="oracle_mut_")
    todo = [(i,) + m for i, m in enumerate(MUTATIONS) if not only or m[0] in only]
    with ThreadPoolExecutor(max_workers=jobs or os.cpu_count() or 1) as ex:
        rows = list(ex.map(lambda t: _one(*t, src, tmp), todo))
    if not quiet:
        for name, _, status, failed, _ in rows:
            print("%-45s %-10s %s" % (name, status, failed), flush=True)
    caught = sum(1 for r in rows if r[2] == "caught")
    equiv = sum(1 for r in rows if r[2] == "equivalent")
    lines = ["# Oracle mutation check (%s)" % time.strftime("%Y-%m-%d"), "",
             "`python scripts/mutate_oracle.py`: each row is one single-line mutation of "
             "`oracle/madpipe_oracle.c`, compiled separately and run against the CPU pins "
             "(%s). **%d / %d caught**, %d equivalent (cannot change any result; see the note)." % (
                 ", ".join("`%s`" % t for t in PIN_TESTS), caught, len(rows) - equiv, equiv), "",
             "| Mutation | Correct line follows | Result | First failing pin |", "|---|---|---|---|"]
    for name, cite, status, failed, dt in rows:
        lines.append("| %s | %s | %s | `%s` |" % (name, cite, status, failed))
    for name, why in EQUIVALENT.items():
        lines += ["", "Equivalent mutant *%s*: %s." % (name, why)]
    open(out, "w").write("\n".join(lines) + "\n")
    print("%d / %d caught, %d equivalent -> %s" % (caught, len(rows) - equiv, equiv, out))
    return caught + equiv == len(rows), rows


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02_oracle_mutations.md"))
    ap.add_argument("--only", nargs="*")
    a = ap.parse_args()
    sys.exit(0 if run(a.out, a.only)[0] else 1)
