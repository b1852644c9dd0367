#!/usr/bin/env python
"""One early-exit GPT solve on cuda:0 (after a warm-up solve), for MADPIPE_PASS_TIMING / profiling of the
time-to-placement path: prints the host wall time of the solve."""
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import chaingen  # noqa: E402
import paper_conf_ipps_beaumontes22_b200 as mp  # noqa: E402
from paper_conf_ipps_beaumontes22_b200 import configs  # noqa: E402

cfg = configs.load("gpt")
ch = chaingen.make(cfg["chain"])
a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
with mp.Context(0, stream=torch.cuda.current_stream().cuda_stream) as ctx:
    ctx.solve(ch, *a, early_exit=True)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    r = ctx.solve(ch, *a, early_exit=True)
    torch.cuda.synchronize()
    print("early-exit solve %.3f ms, j* = %d" % (1e3 * (time.perf_counter() - t0), r["cand_index"]))
