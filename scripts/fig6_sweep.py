"""NEXT row f4: the Figure 6 "dashed line" analogue on synthetic chains.

For a ResNet-50-shaped chain (1000x1000 images, batch 8, fp32 -- P:235) this solves
MadPipe-DP's first phase for every combination of
    M in {3, 4, ..., 16} GB,  P in {2, 4, 8},  beta in {12, 24} GB/s
with the paper's discretisation (11 memory levels, 51 delay levels) and
prints the period of the partitioning found (the "dashed line" of Fig. 6) and the
speed-up U(1,L)/period (Fig. 8's y-axis).  All 84 instances run as ONE batched
sweep (madpipe_solve_batch).  The solid lines (ILP schedules, section 4.3) and
PipeDream are out of scope.

    python scripts/fig6_sweep.py [--n-periods 256] [--out profiles/fig6_resnet50.md]

The paper's qualitative statement checked here: "the period of the partitionings
(the dashed lines) are non-increasing with M" -- on a discretised grid this
is expected but not guaranteed, so violations are reported, not asserted.
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
    ap.add_argument("--n-periods", type=int, default=256)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "fig6_resnet50.md"))
    args = ap.parse_args()
    import numpy as np

    import chaingen
    import paper_conf_ipps_beaumontes22_b200 as mp

    ch = chaingen.resnet50()
    U = float(np.sum(ch["uF"] + ch["uB"]))
    Ms = [g * 10**9 for g in range(3, 17)]
    Ps = [2, 4, 8]
    betas = [12e9, 24e9]
    inst = [(M, P, b) for b in betas for P in Ps for M in Ms]
    with mp.Context(0) as ctx:
        t0 = time.perf_counter()
        res = ctx.solve_batch([ch] * len(inst), [P for _, P, _ in inst], [M for M, _, _ in inst],
                              [b for _, _, b in inst], 11, 51, args.n_periods)
        dt = time.perf_counter() - t0
    lines = ["# Fig. 6-style sweep (dashed lines): ResNet-50-shaped chain, 11 x 51 discretisation",
             "", "%d instances, one madpipe_solve_batch call, %.3f s wall, %d candidate periods each" % (
                 len(inst), dt, args.n_periods), "",
             "period in ms (speed-up U(1,L)/period in brackets); '-' = no feasible period", ""]
    viol = 0
    for b in betas:
        lines.append("## beta = %.0f GB/s" % (b / 1e9))
        lines.append("")
        lines.append("| M (GB) | " + " | ".join("P=%d" % P for P in Ps) + " |")
        lines.append("|---|" + "---|" * len(Ps))
        prev = {P: None for P in Ps}
        for M in Ms:
            cells = []
            for P in Ps:
                r = res[inst.index((M, P, b))]
                if r["cand_index"] < 0:
                    cells.append("-")
                    continue
                per = r["period"]
                if prev[P] is not None and per > prev[P] * (1 + 1e-12):
                    viol += 1
                prev[P] = per
                cells.append("%.1f (%.2fx)" % (per * 1e3, U / per))
            lines.append("| %d | " % (M // 10**9) + " | ".join(cells) + " |")
        lines.append("")
    lines.append("non-monotone steps in M (P:247 expects none): %d" % viol)
    text = "\n".join(lines) + "\n"
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    open(args.out, "w").write(text)
    print(text)


if __name__ == "__main__":
    main()
