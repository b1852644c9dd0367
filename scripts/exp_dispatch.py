#!/usr/bin/env python
"""Experiment: which step kernel wins as a function of P (segment size).  GPT chain (or
argv[1]) with P overridden, n_periods candidates; prints sweep ms per kernel.
Kernel selection is by MADPIPE_KERNEL, read at context creation."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import chaingen
import paper_conf_ipps_beaumontes22_b200 as mp
from paper_conf_ipps_beaumontes22_b200 import configs

cfg = configs.load(sys.argv[1] if len(sys.argv) > 1 else "gpt")
Ps = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "8,16,24,32,40,48,64,96,128").split(",")]
n_c = int(sys.argv[3]) if len(sys.argv) > 3 else 256
ch = chaingen.make(cfg["chain"])
dev = torch.device("cuda", 0)
dchain = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).to(dev) for k in ("uF", "uB", "W", "a")}
for P in Ps:
    out = {"P": P}
    for kern in ("pair", "persist", "v1", "auto"):
        if kern == "auto":
            os.environ.pop("MADPIPE_KERNEL", None)
        else:
            os.environ["MADPIPE_KERNEL"] = kern
        a = (P, cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], n_c)
        with mp.Context(0) as ctx:
            ctx.set_timing(True)
            ctx.solve_dev(dchain, *a)
            r = ctx.solve_dev(dchain, *a)
            out[kern] = round(ctx.last_timing()["sweep_ms"], 2)
            out["cand_" + kern] = r["cand_index"]
    print(json.dumps(out), flush=True)
