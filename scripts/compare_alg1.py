"""NEXT row f1: Algorithm 1 (the paper's serial search around the literal DP) versus
the batched decision-form sweep, on the paper's own setting: ResNet-50-shaped chain
at 1000x1000, batch 8, discretisation 11 memory x 51 delay levels,
101 t_P levels for Algorithm 1, K = 10.

Reports, per (P, M): the periods found, the GPU time-to-placement of each method,
and whether the literal answer is feasible for the decision form (P:199 logic).

    python scripts/compare_alg1.py [--out profiles/r01_alg1_vs_sweep.md]
"""
from __future__ import annotations

import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r01_alg1_vs_sweep.md"))
    ap.add_argument("--n-periods", type=int, default=1024)
    args = ap.parse_args()
    import chaingen
    import paper_conf_ipps_beaumontes22_b200 as mp

    ch = chaingen.resnet50()
    rows = ["# Algorithm 1 (literal DP, K=10) vs batched decision sweep -- ResNet-50-shaped, 11 x 51 levels",
            "", "| P | M (GB) | Alg.1 period (ms) | Alg.1 time (s) | sweep period (ms) | sweep early-exit time (s) "
                "| sweep full time (s) | n_c |", "|---|---|---|---|---|---|---|---|"]
    with mp.Context(0) as ctx:
        ctx.solve(ch, 4, 8 * 10**9, 12e9, 11, 51, 16)      # warm-up (module load, allocations)
        for P in (2, 4, 8):
            for Mg in (4, 8, 16):
                M = Mg * 10**9
                t0 = time.perf_counter()
                a1 = ctx.solve_paper(ch, P, M, 12e9, 11, 51, 101, K=10)
                t1 = time.perf_counter()
                ee = ctx.solve(ch, P, M, 12e9, 11, 51, args.n_periods, early_exit=True)
                t2 = time.perf_counter()
                fu = ctx.solve(ch, P, M, 12e9, 11, 51, args.n_periods)
                t3 = time.perf_counter()
                rows.append("| %d | %d | %s | %.3f | %s | %.3f | %.3f | %d |" % (
                    P, Mg, "%.2f" % (a1["period"] * 1e3) if a1["rc"] == 0 else "-", t1 - t0,
                    "%.2f" % (ee["period"] * 1e3) if ee["rc"] == 0 else "-", t2 - t1, t3 - t2, args.n_periods))
    text = "\n".join(rows) + "\n"
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    open(args.out, "w").write(text)
    print(text)


if __name__ == "__main__":
    main()
