"""Small solves for compute-sanitizer runs (memcheck / racecheck / synccheck).

Covers every kernel the library dispatches:
  * the toy config (step_kernel v1), early_exit=2, a table export;
  * fuzz chains across every NMP template and mode on the default dispatch;
  * the two-layer path (pair_trans / pair_step / pair_fixup): P = 40 and 64 with
    n_mem <= 8 and L >= 4 -- default dispatch (P > 16), plus small fuzz cases with
    MADPIPE_KERNEL=pair forced, a mixed-length solve_batch (tiles of finished
    chains skipped), early_exit = 2, a tiny ring round (MADPIPE_PAIR_ROUND=1:
    every slot its own round, the producer wraps the ring most often);
  * the single-layer persistent kernel (P = 16, as Inception / VGG);
  * the paper-literal DP, the traceback, a small batch.
Run:  compute-sanitizer --tool racecheck python scripts/sanitize_small.py [part ...]
parts: base pair persist literal (default: all)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import chaingen  # noqa: E402
import paper_conf_ipps_beaumontes22_b200 as mp  # noqa: E402
from paper_conf_ipps_beaumontes22_b200 import configs  # noqa: E402

parts = sys.argv[1:] or ["base", "pair", "persist", "literal"]


def ctx_with(**env):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update({k: str(v) for k, v in env.items()})
    try:
        return mp.Context(0)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v


def mem_of(ch, f):
    return int((3 * ch["W"].sum() + 3 * ch["a"].sum()) * f) + 1


rng = np.random.default_rng(5)
if "base" in parts:
    with mp.Context(0) as ctx:
        cfg = configs.load("toy")
        ch = chaingen.make(cfg["chain"])
        a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
        print("toy", ctx.solve(ch, *a)["cand_index"], ctx.solve(ch, *a, early_exit=2)["cand_index"])
        ctx.dp_table(ch, *a, j=3)
        for n_m in (2, 4, 11, 33):
            c2 = chaingen.tiny(rng, 9)
            print("nm", n_m, ctx.solve(c2, 4, mem_of(c2, 0.5), 20.0, n_m, 16, 8)["cand_index"])
        chains = [chaingen.random_chain(1000 + i, L=40) for i in range(3)]
        print("batch", [x["cand_index"] for x in ctx.solve_batch(chains, [4, 6, 9], [10**10, 2 * 10**10, 5 * 10**9],
                                                                  [10e9, 20e9, 50e9], 8, 32, 16)])
if "pair" in parts:
    with mp.Context(0) as ctx:                                   # default dispatch: P > 16 -> pair
        for P, n_m, n_v, L in ((40, 8, 48, 12), (64, 8, 64, 10), (40, 4, 33, 7), (70, 5, 20, 9)):
            c2 = chaingen.tiny(rng, L, a_hi=200)
            r = ctx.solve(c2, P, mem_of(c2, 0.5), 25.0, n_m, n_v, 6)
            print("pair", P, n_m, n_v, L, r["cand_index"], ctx.last_kernel())
            print("pair ee2", ctx.solve(c2, P, mem_of(c2, 0.5), 25.0, n_m, n_v, 9, early_exit=2)["cand_index"])
        Ls = [9, 23, 4, 16, 13]
        chains = [chaingen.tiny(rng, L) for L in Ls]
        res = ctx.solve_batch(chains, [40] * len(Ls), [mem_of(c, 0.5) for c in chains], [30.0] * len(Ls), 8, 24, 5)
        print("pair mixed batch", [x["cand_index"] for x in res], ctx.last_kernel())
    with ctx_with(MADPIPE_KERNEL="pair") as ctx:                 # forced on small P
        for P in (2, 3, 6):
            c2 = chaingen.tiny(rng, 8)
            print("pair forced", P, ctx.solve(c2, P, mem_of(c2, 0.5), 20.0, 8, 16, 6)["cand_index"])
    os.environ["MADPIPE_PAIR_ROUND"] = "1"                      # one slot per producer round (read per launch)
    with mp.Context(0) as ctx:
        c2 = chaingen.tiny(rng, 14)
        print("pair round1", ctx.solve(c2, 40, mem_of(c2, 0.5), 25.0, 8, 40, 5)["cand_index"])
    del os.environ["MADPIPE_PAIR_ROUND"]
if "persist" in parts:
    with mp.Context(0) as ctx:
        for P, n_m, n_v, L in ((16, 8, 128, 10), (16, 8, 40, 6)):
            c2 = chaingen.tiny(rng, L)
            print("persist", ctx.solve(c2, P, mem_of(c2, 0.5), 25.0, n_m, n_v, 5)["cand_index"], ctx.last_kernel())
if "literal" in parts:
    with mp.Context(0) as ctx:
        r = chaingen.resnet50()
        print("resnet paper grid", ctx.solve(r, 4, 8 * 10**9, 12e9, 11, 51, 16)["cand_index"])
        print("literal", ctx.solve_paper({k: (v[:21] if k == "a" else v[:20]) if k != "name" else v
                                          for k, v in r.items()}, 3, 6 * 10**9, 12e9, 11, 17, 11, K=3)["period"])
print("sanitize-run done")
