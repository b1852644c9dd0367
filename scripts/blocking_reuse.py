#!/usr/bin/env python
"""Source-row reuse vs in-block options for 2-, 3- and 4-layer blocking, measured on the oracle's GPT
tables (analysis behind profiles/r02b_step_bounds.md; calls oracle/ only, no GPU):

    python scripts/blocking_reuse.py <candidate j>

For three passes (first layers 41, 121, 201) and every v-tile of B layers x VB delay rows (rows of layer
l0+i shifted by round((U(l0+i) - U(l0)) / dV) levels, the two-layer kernel's alignment), it counts the
useful (row, source row) visits whose source slab is final before the pass (k <= l0), the distinct
source rows (k, v') they read (what a tile loads), and the in-block visits (k > l0, which need a fixup).
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import chaingen  # noqa: E402
import oracle  # noqa: E402

cfg = json.load(open(os.path.join(ROOT, "configs", "gpt.json")))
ch = chaingen.gpt()
P, M, beta, nm, nv, nc = cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"]
pr = oracle.prep(ch, P, beta)
Up, L = pr["Up"], len(ch["uF"])
Wp = np.concatenate([[0], np.cumsum(np.array(ch["W"], dtype=np.int64))])
j = int(sys.argv[1]) if len(sys.argv) > 1 else 150
tau = pr["lb"] + j * ((pr["ub"] - pr["lb"]) / (nc - 1))
dV = (Up[L] + pr["SC"]) / (nv - 1)
A, _, _ = oracle.table(ch, P, M, beta, nm, nv, 0, tau, with_arg=False)
finite_row = np.isfinite(A).any(axis=(1, 3))          # [l][v]


def window(l):
    return [k for k in range(1, l + 1) if Up[l] - Up[k - 1] <= tau and 3 * (Wp[l] - Wp[k - 1]) <= M]


for B, VB in [(2, 4), (3, 3), (4, 2)]:
    visits = loaded = inblock = 0
    for l0 in (41, 121, 201):
        shifts = [int(np.rint((Up[l0 + i] - Up[l0]) / dV)) for i in range(B)]
        for vt in range(-(20 // VB), nv // VB + 1):
            rows = [(l0 + i, vt * VB - shifts[i] + r) for i in range(B) for r in range(VB)]
            sources = set()
            for lr, v in rows:
                if not 0 <= v < nv:
                    continue
                for k in window(lr):
                    _, nf, d, vn = oracle.transition(ch, P, M, beta, nm, nv, 0, tau, k, lr, v)
                    if not 0 <= vn <= nv - 1 or (not nf and d > nm - 1) or not finite_row[k - 1][vn]:
                        continue
                    if k > l0:
                        inblock += 1
                        continue
                    visits += 1
                    sources.add((k, vn))
            loaded += len(sources)
    layers = 3 * B
    print("B=%d VB=%d: reuse %.2f, source rows loaded per layer %d, in-block visits per layer %d"
          % (B, VB, visits / loaded, loaded // layers, inblock // layers), flush=True)
