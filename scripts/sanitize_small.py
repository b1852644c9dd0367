"""Small solves for compute-sanitizer runs (memcheck / racecheck / synccheck): the toy
config, a few fuzz cases across all NMP templates and modes, ResNet-50 with the paper
discretisation, the literal DP, and a small batch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import chaingen  # noqa: E402
import paper_conf_ipps_beaumontes22_b200 as mp  # noqa: E402
from paper_conf_ipps_beaumontes22_b200 import configs  # noqa: E402

with mp.Context(0) as ctx:
    cfg = configs.load("toy")
    ch = chaingen.make(cfg["chain"])
    a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    print(ctx.solve(ch, *a)["cand_index"], ctx.solve(ch, *a, early_exit=2)["cand_index"])
    ctx.dp_table(ch, *a, j=3)
    rng = np.random.default_rng(5)
    for n_m in (2, 4, 11, 33):
        c2 = chaingen.tiny(rng, 9)
        M = int((3 * c2["W"].sum() + 3 * c2["a"].sum()) * 0.5)
        print(n_m, ctx.solve(c2, 4, M, 20.0, n_m, 16, 8)["cand_index"])
    r = chaingen.resnet50()
    print(ctx.solve(r, 4, 8 * 10**9, 12e9, 11, 51, 16)["cand_index"])
    print(ctx.solve_paper({k: (v[:21] if k == "a" else v[:20]) if k != "name" else v for k, v in r.items()},
                          3, 6 * 10**9, 12e9, 11, 17, 11, K=3)["period"])
    chains = [chaingen.random_chain(1000 + i, L=40) for i in range(3)]
    print([x["cand_index"] for x in ctx.solve_batch(chains, [4, 6, 9], [10**10, 2 * 10**10, 5 * 10**9],
                                                      [10e9, 20e9, 50e9], 8, 32, 16)])
print("sanitize-run done")
