#!/usr/bin/env python
"""One full GPT candidate sweep (madpipe_sweep, rank 0 of 1: the sweep without the
winner re-solve) on cuda:0, for an ncu DRAM-traffic capture of every step-kernel
launch; writes the sweep's algorithmic byte counts to the JSON path given."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import chaingen  # noqa: E402
import paper_conf_ipps_beaumontes22_b200 as mp  # noqa: E402
from paper_conf_ipps_beaumontes22_b200 import configs  # noqa: E402

cfg = configs.load("gpt")
ch = chaingen.make(cfg["chain"])
d = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).cuda() for k in ("uF", "uB", "W", "a")}
a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
jl = torch.empty(1, dtype=torch.int32, device="cuda")
with mp.Context(0, stream=torch.cuda.current_stream().cuda_stream) as ctx:
    cu = ctx.sweep(d, *a, 0, 1, jl.data_ptr())
    sb = ctx.last_step_bytes()
    S = cfg["n_delay"] * cfg["n_mem"]
    out = dict(cell_updates=cu, moved_bytes=sb["load_bytes"] + sb["store_bytes"], segments=sb["segments"],
               compulsory_bytes=2 * (cfg["L"] + 1) * cfg["P"] * S * 8 * cfg["n_periods"],
               kernel=ctx.last_kernel(), j_local=int(jl.item()))
json.dump(out, open(sys.argv[1] if len(sys.argv) > 1 else "one_sweep.json", "w"), indent=1)
print(json.dumps(out))
