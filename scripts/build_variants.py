#!/usr/bin/env python
"""Build the compile-time A/B variants of libmadpipe as their own in-tree libraries
(paper_conf_ipps_beaumontes22_b200/libmadpipe_<name>.so, flags stamped in <lib>.flags),
for scripts/gpu_ab.sh.  Every variant must pass the pair-path parity tests before
it is timed; the defaults in the sources are the variants that won.

    python scripts/build_variants.py [name ...]      (default: all)
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
VARIANTS = {
    "base": "",                                   # the defaults
    "qatomic": "-DMP_QUEUE_ATOMIC=1",             # queue words through shared atomics (racecheck-clean)
    "prof": "-DMP_PAIR_PROF=1",                   # MADPIPE_PROF=1 cycle counters compiled in (1.8% slower)
    "poll0": "-DMP_POLL_NS=0",                    # consumers spin without back-off
    "poll100": "-DMP_POLL_NS=100",
    "tworow": "-DMP_PAIR_ONEROW=0",               # always relax both processor rows of a thread
    "nol2pf": "-DMP_PAIR_L2PF=0",                 # no L2 prefetch of list entries ahead of the producer
    "l2pf6": "-DMP_PAIR_L2PF=6",                  # L2 prefetch 6 rounds ahead
    "l2pf2": "-DMP_PAIR_L2PF=2",
    "l2pf4": "-DMP_PAIR_L2PF=4",
    "tminb6": "-DMP_TRANS_MINB=6",                # list builder compiled for 6 resident blocks per SM (80 registers)
    "tminb4": "-DMP_TRANS_MINB=4",
    "fixminb1": "-DMP_FIX_MINB=1",                # fixup without a residency target (72 registers, 7 blocks per SM)
    "ctas3": "-DMP_PAIR_CTAS=3",                  # 3 CTAs per SM (16-slot rings, <= 75 registers)
    # MADPIPE_REPLAY=pass,reps,diag honoured (diag 1: consumers skip the relaxation, 2: producer
    # skips the copies, 3: both) -- diagnostic replays only, never the solve itself
    "diag": "-DMP_DIAG=1",
}

if __name__ == "__main__":
    names = sys.argv[1:] or list(VARIANTS)
    for n in names:
        lib = os.path.join(ROOT, "paper_conf_ipps_beaumontes22_b200", "libmadpipe_%s.so" % n)
        env = dict(os.environ, MADPIPE_DEFS=VARIANTS[n], MADPIPE_LIB=lib)
        subprocess.check_call([sys.executable, "-c", "from paper_conf_ipps_beaumontes22_b200 import build; "
                               "print(build.build(force=True))"], cwd=ROOT, env=env)
        print(n, VARIANTS[n] or "(defaults)")
