"""ctypes binding of libmadpipe.so (include/madpipe.h).  Argument marshalling only:
every step of the DP runs in the library's CUDA kernels.  There is no CPU
fallback: if the library is missing or no GPU is usable, calls raise."""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# MADPIPE_LIB: an alternative in-tree build (A/B experiments, build.py MADPIPE_DEFS)
LIB_PATH = os.environ.get("MADPIPE_LIB") or os.path.join(_HERE, "libmadpipe.so")

OK, INFEASIBLE, EINVAL, ENOMEM, ECUDA, ENCCL, ESTATE = 0, 1, -1, -2, -3, -4, -5
VRANGE_PAPER, VRANGE_SAFE = 0, 1

_i32p = ctypes.POINTER(ctypes.c_int32)
_i64p = ctypes.POINTER(ctypes.c_int64)
_dp = ctypes.POINTER(ctypes.c_double)


class Chain(ctypes.Structure):
    _fields_ = [("L", ctypes.c_int32), ("uF", ctypes.c_void_p), ("uB", ctypes.c_void_p),
                ("W", ctypes.c_void_p), ("a", ctypes.c_void_p)]


class Disc(ctypes.Structure):
    _fields_ = [("n_mem", ctypes.c_int32), ("n_delay", ctypes.c_int32),
                ("n_periods", ctypes.c_int32), ("v_range", ctypes.c_int32),
                ("early_exit", ctypes.c_int32)]


class Op(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("stage", ctypes.c_int32), ("group", ctypes.c_int32),
                ("f_shift", ctypes.c_int32), ("b_shift", ctypes.c_int32), ("pad_", ctypes.c_int32),
                ("f_start", ctypes.c_double), ("f_len", ctypes.c_double), ("b_start", ctypes.c_double),
                ("b_len", ctypes.c_double)]


class Alloc(ctypes.Structure):
    _fields_ = [("period", ctypes.c_double), ("load_period", ctypes.c_double),
                ("special_load", ctypes.c_double), ("cand_index", ctypes.c_int32),
                ("n_stages", ctypes.c_int32), ("stage_first", _i32p), ("stage_last", _i32p),
                ("stage_proc", _i32p), ("cell_updates", ctypes.c_int64)]


_lib = None


def lib():
    """Load libmadpipe.so; raise loudly if it was not built (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError("libmadpipe.so not built at %s -- run __graft_entry__.build() "
                          "(there is no CPU fallback)" % LIB_PATH)
    L = ctypes.CDLL(LIB_PATH)
    vp = ctypes.c_void_p
    cp = ctypes.POINTER(Chain)
    dcp = ctypes.POINTER(Disc)
    ap = ctypes.POINTER(Alloc)
    sig = {
        "madpipe_get_unique_id": (ctypes.c_int, [ctypes.c_char_p]),
        "madpipe_ctx_create": (ctypes.c_int, [ctypes.POINTER(vp), ctypes.c_int, ctypes.c_int32, ctypes.c_int32,
                                              ctypes.c_char_p, vp, ctypes.c_int64]),
        "madpipe_ctx_info": (ctypes.c_int, [vp, _i32p, _i32p, _i32p]),
        "madpipe_ctx_destroy": (None, [vp]),
        "madpipe_last_error": (ctypes.c_char_p, [vp]),
        "madpipe_validate": (ctypes.c_int, [cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double, dcp]),
        "madpipe_shard": (ctypes.c_int, [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, _i32p, _i32p]),
        "madpipe_cell_updates": (ctypes.c_int64, [cp, ctypes.c_int32, dcp, ctypes.c_double]),
        "madpipe_solve": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double, dcp, ap]),
        "madpipe_solve_dev": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double, dcp, ap]),
        "madpipe_sweep": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double, dcp,
                                         ctypes.c_int32, ctypes.c_int32, vp, _i64p]),
        "madpipe_resolve": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double, dcp,
                                           vp, ap]),
        "madpipe_solve_batch": (ctypes.c_int, [vp, ctypes.c_int32, cp, _i32p, _i64p, _dp, dcp, ap]),
        "madpipe_sweep_batch": (ctypes.c_int, [vp, ctypes.c_int32, cp, _i32p, _i64p, _dp, dcp, ctypes.c_int32,
                                               ctypes.c_int32, _i32p, _i64p]),
        "madpipe_resolve_batch": (ctypes.c_int, [vp, ctypes.c_int32, cp, _i32p, _i64p, _dp, dcp, _i32p,
                                                 ctypes.c_int32, ctypes.c_int32, ap]),
        "madpipe_batch_plan": (ctypes.c_int, [ctypes.c_int32, cp, _i32p, _dp, dcp, ctypes.c_int32, _i32p, _i64p,
                                              _i64p]),
        "madpipe_resolve_plan": (ctypes.c_int, [ctypes.c_int32, cp, _i32p, _dp, dcp, _i32p, ctypes.c_int32,
                                                _i32p]),
        "madpipe_candidates": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double,
                                              dcp, _dp, _dp]),
        "madpipe_dp_table": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double,
                                            dcp, ctypes.c_int32, _dp, _i32p]),
        "madpipe_last_timing": (ctypes.c_int, [vp, _dp, _dp, _i64p]),
        "madpipe_set_timing": (ctypes.c_int, [vp, ctypes.c_int]),
        "madpipe_last_io": (ctypes.c_int, [vp, _i64p, _i64p]),
        "madpipe_last_counts": (ctypes.c_int, [vp, _i64p, _i64p, _i64p]),
        "madpipe_last_step_bytes": (ctypes.c_int, [vp, _i64p, _i64p, _i64p]),
        "madpipe_last_kernel": (ctypes.c_int, [vp, _i32p]),
        "madpipe_solve_paper": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double,
                                               ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ap,
                                               _dp, _dp]),
        "madpipe_literal_table": (ctypes.c_int, [vp, cp, ctypes.c_int32, ctypes.c_int64, ctypes.c_double,
                                                 ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_double,
                                                 _dp, _i32p]),
        "madpipe_schedule": (ctypes.c_int, [cp, ctypes.c_double, ctypes.c_double, ctypes.c_int32, _i32p, _i32p,
                                            ctypes.POINTER(Op), _i32p]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return _lib


EXPORTED = ["madpipe_get_unique_id", "madpipe_ctx_create", "madpipe_ctx_destroy", "madpipe_ctx_info",
            "madpipe_last_error", "madpipe_validate",
            "madpipe_shard", "madpipe_cell_updates", "madpipe_solve", "madpipe_solve_dev",
            "madpipe_sweep", "madpipe_resolve", "madpipe_solve_batch", "madpipe_sweep_batch",
            "madpipe_resolve_batch", "madpipe_batch_plan", "madpipe_resolve_plan", "madpipe_candidates",
            "madpipe_dp_table", "madpipe_last_timing", "madpipe_set_timing", "madpipe_last_io",
            "madpipe_last_counts", "madpipe_last_step_bytes", "madpipe_last_kernel", "madpipe_schedule", "madpipe_solve_paper", "madpipe_literal_table"]


class MadpipeError(RuntimeError):
    def __init__(self, rc, msg):
        super().__init__("libmadpipe rc=%d: %s" % (rc, msg))
        self.rc = rc


def last_error(ctx=None) -> str:
    s = lib().madpipe_last_error(ctx)
    return s.decode() if s else ""


def check(rc, ctx=None, allow_infeasible=True):
    if rc == OK or (allow_infeasible and rc == INFEASIBLE):
        return rc
    raise MadpipeError(rc, last_error(ctx))


class HostChain:
    """Keeps contiguous numpy copies alive for the duration of a call."""

    def __init__(self, ch):
        self.uF = np.ascontiguousarray(ch["uF"], dtype=np.float64)
        self.uB = np.ascontiguousarray(ch["uB"], dtype=np.float64)
        self.W = np.ascontiguousarray(ch["W"], dtype=np.int64)
        self.a = np.ascontiguousarray(ch["a"], dtype=np.int64)
        self.L = len(self.uF)
        if len(self.uB) != self.L or len(self.W) != self.L or len(self.a) != self.L + 1:
            raise ValueError("chain arrays must have lengths L, L, L, L+1")
        self.c = Chain(self.L, self.uF.ctypes.data, self.uB.ctypes.data, self.W.ctypes.data,
                       self.a.ctypes.data)


def make_disc(n_mem, n_delay, n_periods, v_range=VRANGE_PAPER, early_exit=False) -> Disc:
    ee = int(early_exit) if not isinstance(early_exit, bool) else (1 if early_exit else 0)
    return Disc(int(n_mem), int(n_delay), int(n_periods), int(v_range), ee)


class AllocBuf:
    def __init__(self, L):
        self.first = np.zeros(max(L, 1), np.int32)
        self.last = np.zeros(max(L, 1), np.int32)
        self.proc = np.zeros(max(L, 1), np.int32)
        self.s = Alloc(0.0, 0.0, 0.0, -1, 0, self.first.ctypes.data_as(_i32p),
                       self.last.ctypes.data_as(_i32p), self.proc.ctypes.data_as(_i32p), 0)

    def result(self, rc):
        n = self.s.n_stages
        return dict(rc=rc, period=self.s.period, load_period=self.s.load_period,
                    special_load=self.s.special_load, cand_index=self.s.cand_index,
                    stages=[(int(self.first[i]), int(self.last[i]), int(self.proc[i])) for i in range(n)],
                    cell_updates=int(self.s.cell_updates))
