"""Build libmadpipe.so in-tree with nvcc for sm_100a (no JIT, no torch extension).

Flags: -gencode arch=compute_100a,code=sm_100a; --fmad=false and explicit
__d*_rn intrinsics keep every fp64 rounding identical to the CPU oracle;
-Xcompiler -ffp-contract=off does the same for host code; -lineinfo maps ncu
source pages to the kernels.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.environ.get("MADPIPE_LIB") or os.path.join(HERE, "libmadpipe.so")
SOURCES = ["mp_kernels.cu", "mp_step_persist.cu", "mp_step_pair.cu", "mp_api.cu", "mp_schedule.cu", "mp_literal.cu", "mp_comm.cu"]
HEADERS = ["mp_internal.cuh", "mp_device.cuh", os.path.join("..", "..", "include", "madpipe.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "--fmad=false", "-Xcompiler", "-fPIC,-ffp-contract=off",
         "-Xptxas", "-v"] + os.environ.get("MADPIPE_DEFS", "").split()   # A/B experiment macros


def _defs_stamp() -> str:
    return " ".join(FLAGS)


def _stale() -> bool:
    """Rebuild when a source is newer than the library or when the library was built
    with other flags (MADPIPE_DEFS variants: the flags are stamped next to it)."""
    if not os.path.exists(LIB):
        return True
    stamp = LIB + ".flags"
    if not os.path.exists(stamp) or open(stamp).read() != _defs_stamp():
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.abspath(__file__)]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    objs = []
    for src in SOURCES:
        obj = LIB + "." + src.replace(".cu", ".o")
        cmd = [NVCC, *ARCH, *FLAGS, "-c", os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError("nvcc failed for %s" % src)
        if verbose:
            sys.stderr.write(r.stderr)
        objs.append(obj)
    tmp = LIB + ".tmp.%d" % os.getpid()
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart_static", "-lrt", "-ldl", "-lpthread"]   # NCCL: dlopen (mp_comm.cu)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc link failed")
    os.replace(tmp, LIB)
    with open(LIB + ".flags", "w") as f:
        f.write(_defs_stamp())
    for o in objs:
        os.remove(o)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
