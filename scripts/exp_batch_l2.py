#!/usr/bin/env python
"""Experiment: does a small batch (few candidates in lockstep) make layer l+1's source
reads hit L2 (layer l read ~94% of the same rows)?  Full GPT sweep with the table budget
capped to B candidates per batch; prints sweep time and the summed step-kernel time."""
import json, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import chaingen
import paper_conf_ipps_beaumontes22_b200 as mp
from paper_conf_ipps_beaumontes22_b200 import configs

cfg = configs.load(sys.argv[1] if len(sys.argv) > 1 else "gpt")
ch = chaingen.make(cfg["chain"])
dev = torch.device("cuda", 0)
dchain = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).to(dev) for k in ("uF", "uB", "W", "a")}
a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
nmp = 1
while nmp < cfg["n_mem"]:
    nmp *= 2
tbytes = (cfg["L"] + 1) * cfg["n_delay"] * cfg["P"] * nmp * 8
for B in [int(x) for x in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["0", "64", "16", "8", "4", "2"])]:
    with mp.Context(0, mem_budget=(B * ((tbytes + 255) // 256 * 256) if B else 0)) as ctx:
        ctx.set_timing(os.environ.get("EXP_NO_LAUNCH_TIMING") is None)
        ctx.solve_dev(dchain, *a)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = ctx.solve_dev(dchain, *a)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        tm = ctx.last_timing(); cn = ctx.last_counts(); sb = ctx.last_step_bytes()
        print(json.dumps(dict(batch=B or "default", wall_s=dt, sweep_ms=tm["sweep_ms"], step_ms=tm["step_ms"],
                              launches=tm["launches"], useful=cn["useful_updates"],
                              useful_TBps_step=cn["useful_updates"] * 8 / (tm["step_ms"] * 1e-3) / 1e12,
                              cand=r["cand_index"], load_GB=sb["load_bytes"] / 1e9,
                              store_GB=sb["store_bytes"] / 1e9, segments=sb["segments"],
                              step_TBps_algo=(sb["load_bytes"] + sb["store_bytes"]) / (tm["step_ms"] * 1e-3) / 1e12)),
              flush=True)
