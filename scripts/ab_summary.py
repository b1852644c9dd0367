#!/usr/bin/env python
"""Summarise a gpu_ab.sh run: ms per solve and step-kernel ms per variant/round, the
MADPIPE_PROF counters and the diagnostic replays."""
import glob
import json
import os

OUT = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "gpurun_out")
for f in sorted(glob.glob(os.path.join(OUT, "ab_*_r*_[12].json"))):
    try:
        d = json.load(open(f))
        print("%-28s solve %7.1f ms  step kernel %7.1f ms  match %s" % (
            os.path.basename(f), d["ms_per_step"], d["roofline"]["kernel_ms_per_step"],
            d["result"].get("matches_oracle")))
    except Exception as e:  # noqa: BLE001
        print(os.path.basename(f), "ERR", e)
for f in sorted(glob.glob(os.path.join(OUT, "ab_prof.err"))):
    for ln in open(f):
        if "prof pair" in ln:
            print(ln.strip()[:260])
            break
for f in sorted(glob.glob(os.path.join(OUT, "ab_r64_*.txt"))):
    print(os.path.basename(f), " ".join(ln.split()[-4] for ln in open(f)))
