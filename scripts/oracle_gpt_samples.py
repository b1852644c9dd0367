#!/usr/bin/env python
"""Write configs/gpt_oracle_samples.json: oracle values of stratified GPT candidates.

Calls only chaingen and oracle/ (every stored value comes from the CPU oracle).
For each sampled candidate j of the GPT config (j <= j*, j*+1..8,
16 stratified above, plus 511 / 767 / 1023): the root A_j[L][P-1][0][0], the
cell-update count, the oracle's single-thread time, and a SHA-256 digest of two
whole slabs of the table (l = L/2 and l = L, float64 bytes in [p][v][m] order),
so the GPU test can check every cell of those slabs without the oracle.

    python scripts/oracle_gpt_samples.py [--procs 8]
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import sys
import time
from concurrent.futures import ProcessPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import chaingen  # noqa: E402
import oracle  # noqa: E402
from paper_conf_ipps_beaumontes22_b200 import configs  # noqa: E402

OUT = os.path.join(ROOT, "configs", "gpt_oracle_samples.json")


def sample_js(jstar, n_c):
    js = set(range(0, jstar + 1)) | set(range(jstar + 1, min(jstar + 9, n_c)))
    lo = jstar + 9
    if lo < n_c:
        for i in range(16):
            js.add(int(round(lo + i * (n_c - 1 - lo) / 15.0)))
    js |= {511, 767, n_c - 1}
    return sorted(j for j in js if 0 <= j < n_c)


def one(j):
    cfg = configs.load("gpt")
    ch = chaingen.make(cfg["chain"])
    tau = oracle.solve(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"],
                       j_lo=0, j_hi=1)["tau"]
    t0 = time.perf_counter()
    A, _, cu = oracle.table(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["v_range"],
                            tau[j], with_arg=False)
    dt = time.perf_counter() - t0
    L = cfg["L"]
    digests = {str(l): hashlib.sha256(A[l].tobytes()).hexdigest() for l in (L // 2, L)}
    return dict(j=j, tau=float(tau[j]).hex(), root=float(A[L, cfg["P"] - 1, 0, 0]).hex(), cell_updates=int(cu),
                oracle_s=dt, slab_sha256=digests, finite_root_slab=int(__import__("numpy").isfinite(A[L]).sum()))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--procs", type=int, default=os.cpu_count() or 1)
    a = ap.parse_args()
    cfg = configs.load("gpt")
    js = sample_js(cfg["oracle_cand_index"], cfg["n_periods"])
    # longest first (the windows, hence the cost, grow with j)
    with ProcessPoolExecutor(a.procs) as ex:
        rows = list(ex.map(one, sorted(js, reverse=True)))
    rows.sort(key=lambda r: r["j"])
    json.dump({"config": "gpt", "digest": cfg["digest"], "oracle_cand_index": cfg["oracle_cand_index"],
               "note": "written by scripts/oracle_gpt_samples.py from oracle/ only; floats as hex",
               "samples": rows}, open(OUT, "w"), indent=1)
    print("wrote %d samples -> %s" % (len(rows), OUT))


if __name__ == "__main__":
    main()
