"""CPU oracle for the MadPipe memory-aware DP -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ipps_beaumontes22_b200``) never imports it and
shares no code with it.

Contents
--------
* ``madpipe_oracle.c`` -- the plain decision DP (steps
  O1-O9), compiled with ``gcc -O2 -ffp-contract=off -fopenmp`` into
  ``liboracle.so`` and called through ctypes below.
* ``bruteforce.py``   -- O11/O12: exhaustive enumeration of partitions and
  assignments on tiny chains (pure Python, independent of the C file).
* ``simulator.py``    -- O10: 1F1B* grouping/pattern simulator
  and the memory / load checks of returned allocations.
* ``special.py``      -- O13: closed forms and an independent max-coverage DP
  for the memory-free special case.

Parity with numbers printed in the paper is UNPINNED: the paper prints no
worked example (figures stripped: P:209).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "madpipe_oracle.c")
# ORACLE_LIB: a prebuilt alternative (only scripts/mutate_oracle.py uses it, to run the
# pins against deliberately broken copies of madpipe_oracle.c)
_LIB = os.environ.get("ORACLE_LIB") or os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

PAPER = 0
SAFE = 1

OK = 0
INFEASIBLE = 1


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain C, no FMA contraction, OpenMP over candidates)."""
    if os.environ.get("ORACLE_LIB"):
        return _LIB
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        cmd = ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
               "-fPIC", "-shared", "-Wall", "-o", tmp, _SRC, "-lm"]
        subprocess.check_call(cmd)
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            dp = ctypes.POINTER(ctypes.c_double)
            ip = ctypes.POINTER(ctypes.c_int64)
            i32p = ctypes.POINTER(ctypes.c_int32)
            cint = ctypes.c_int
            L.oracle_oplus.restype = ctypes.c_double
            L.oracle_oplus.argtypes = [ctypes.c_double] * 3
            L.oracle_mem.restype = ctypes.c_int64
            L.oracle_mem.argtypes = [cint, ip, ip, cint, cint, ctypes.c_int64]
            L.oracle_prep.restype = cint
            L.oracle_prep.argtypes = [cint, dp, dp, ip, ip, cint, ctypes.c_double,
                                      dp, ip, ip, dp, dp, dp, dp]
            L.oracle_transition.restype = cint
            L.oracle_transition.argtypes = [cint, dp, dp, ip, ip, cint, ctypes.c_int64,
                                            ctypes.c_double, cint, cint, cint, ctypes.c_double,
                                            cint, cint, cint, ip, i32p, ip, i32p]
            L.oracle_table.restype = cint
            L.oracle_table.argtypes = [cint, dp, dp, ip, ip, cint, ctypes.c_int64, ctypes.c_double,
                                       cint, cint, cint, ctypes.c_double, dp, i32p, ip]
            L.oracle_solve.restype = cint
            L.oracle_solve.argtypes = [cint, dp, dp, ip, ip, cint, ctypes.c_int64, ctypes.c_double,
                                       cint, cint, cint, cint, cint, cint, cint, cint,
                                       dp, dp, dp, dp, dp, i32p, i32p, i32p, i32p, i32p, ip]
            L.oracle_literal_table.restype = cint
            L.oracle_literal_table.argtypes = [cint, dp, dp, ip, ip, cint, ctypes.c_int64, ctypes.c_double,
                                               cint, cint, cint, ctypes.c_double, dp, i32p]
            L.oracle_literal_solve.restype = cint
            L.oracle_literal_solve.argtypes = [cint, dp, dp, ip, ip, cint, ctypes.c_int64, ctypes.c_double,
                                               cint, cint, cint, cint, dp, dp, dp, i32p, i32p, i32p, i32p, i32p]
            _lib = L
    return _lib


def _d(x):
    return np.ascontiguousarray(x, dtype=np.float64)


def _i(x):
    return np.ascontiguousarray(x, dtype=np.int64)


def _ptr(arr, t):
    return arr.ctypes.data_as(ctypes.POINTER(t))


def _chain_args(ch):
    uF, uB, W, a = _d(ch["uF"]), _d(ch["uB"]), _i(ch["W"]), _i(ch["a"])
    L = len(uF)
    assert len(uB) == L and len(W) == L and len(a) == L + 1
    keep = (uF, uB, W, a)
    return L, keep, (_ptr(uF, ctypes.c_double), _ptr(uB, ctypes.c_double),
                     _ptr(W, ctypes.c_int64), _ptr(a, ctypes.c_int64))


def oplus(x: float, y: float, tau: float) -> float:
    """x (+) y of P:177."""
    return lib().oracle_oplus(x, y, tau)


def mem(W, a, k: int, l: int, g: int) -> int:
    """M(k, l, g) of P:159 (int64 bytes)."""
    W, a = _i(W), _i(a)
    return lib().oracle_mem(len(W), _ptr(W, ctypes.c_int64), _ptr(a, ctypes.c_int64), k, l, g)


def prep(ch, P: int, beta: float):
    L, keep, ptrs = _chain_args(ch)
    Up = np.zeros(L + 1); Wp = np.zeros(L + 1, np.int64); Ap = np.zeros(L + 1, np.int64)
    C = np.zeros(L + 1); SC = ctypes.c_double(); lb = ctypes.c_double(); ub = ctypes.c_double()
    rc = lib().oracle_prep(L, *ptrs, P, beta, _ptr(Up, ctypes.c_double), _ptr(Wp, ctypes.c_int64),
                           _ptr(Ap, ctypes.c_int64), _ptr(C, ctypes.c_double), ctypes.byref(SC),
                           ctypes.byref(lb), ctypes.byref(ub))
    if rc:
        raise ValueError("oracle_prep rc=%d" % rc)
    return dict(Up=Up, Wp=Wp, Ap=Ap, C=C, SC=SC.value, lb=lb.value, ub=ub.value)


def transition(ch, P, M, beta, n_m, n_v, v_range, tau, k, l, v):
    L, keep, ptrs = _chain_args(ch)
    g = ctypes.c_int64(); nf = ctypes.c_int32(); d = ctypes.c_int64(); vn = ctypes.c_int32()
    rc = lib().oracle_transition(L, *ptrs, P, M, beta, n_m, n_v, v_range, tau, k, l, v,
                                 ctypes.byref(g), ctypes.byref(nf), ctypes.byref(d), ctypes.byref(vn))
    if rc:
        raise ValueError("oracle_transition rc=%d" % rc)
    return g.value, bool(nf.value), d.value, vn.value


def table(ch, P, M, beta, n_m, n_v, v_range, tau, with_arg=True):
    """Full DP table at period tau: (A[l][p][v][m], ARG or None, cell_updates)."""
    L, keep, ptrs = _chain_args(ch)
    A = np.empty((L + 1, P, n_v, n_m), np.float64)
    ARG = np.empty((L + 1, P, n_v, n_m), np.int32) if with_arg else None
    cu = ctypes.c_int64()
    rc = lib().oracle_table(L, *ptrs, P, M, beta, n_m, n_v, v_range, tau, _ptr(A, ctypes.c_double),
                            _ptr(ARG, ctypes.c_int32) if with_arg else None, ctypes.byref(cu))
    if rc:
        raise ValueError("oracle_table rc=%d" % rc)
    return A, ARG, cu.value


def solve(ch, P, M, beta, n_m, n_v, n_c, v_range=PAPER, early_exit=False, j_lo=0, j_hi=None,
          n_threads=1):
    """Candidate sweep (O3-O9).  Returns a dict (rc, period, load_period, special_load,
    cand_index, stages=[(first,last,proc)], cell_updates, tau[n_c], root[n_c])."""
    L, keep, ptrs = _chain_args(ch)
    if j_hi is None:
        j_hi = n_c
    tau = np.empty(n_c); root = np.empty(n_c)
    period = ctypes.c_double(); lp = ctypes.c_double(); sl = ctypes.c_double()
    ci = ctypes.c_int32(); ns = ctypes.c_int32(); cu = ctypes.c_int64()
    sf = np.zeros(L, np.int32); sl_ = np.zeros(L, np.int32); sp = np.zeros(L, np.int32)
    rc = lib().oracle_solve(L, *ptrs, P, M, beta, n_m, n_v, v_range, n_c, j_lo, j_hi,
                            1 if early_exit else 0, n_threads,
                            _ptr(tau, ctypes.c_double), _ptr(root, ctypes.c_double),
                            ctypes.byref(period), ctypes.byref(lp), ctypes.byref(sl), ctypes.byref(ci),
                            ctypes.byref(ns), _ptr(sf, ctypes.c_int32), _ptr(sl_, ctypes.c_int32),
                            _ptr(sp, ctypes.c_int32), ctypes.byref(cu))
    if rc < 0:
        raise ValueError("oracle_solve rc=%d" % rc)
    n = ns.value
    return dict(rc=rc, period=period.value, load_period=lp.value, special_load=sl.value,
                cand_index=ci.value,
                stages=[(int(sf[i]), int(sl_[i]), int(sp[i])) for i in range(n)],
                cell_updates=cu.value, tau=tau, root=root)


def literal_table(ch, P, M, beta, n_m, n_v, n_t, That, with_arg=True):
    """NEXT row f1: the paper-literal DP table T(l, p, t, v, m) at target That (layout
    [l][p][t][v][m]) and its decisions."""
    L, keep, ptrs = _chain_args(ch)
    A = np.empty((L + 1, P, n_t, n_v, n_m), np.float64)
    ARG = np.empty((L + 1, P, n_t, n_v, n_m), np.int32) if with_arg else None
    rc = lib().oracle_literal_table(L, *ptrs, P, M, beta, n_m, n_v, n_t, That, _ptr(A, ctypes.c_double),
                                    _ptr(ARG, ctypes.c_int32) if with_arg else None)
    if rc:
        raise ValueError("oracle_literal_table rc=%d" % rc)
    return A, ARG


def literal_solve(ch, P, M, beta, n_m, n_v, n_t, K=10):
    """NEXT row f1: Algorithm 1 (reading Q15) around the literal DP."""
    L, keep, ptrs = _chain_args(ch)
    T = np.empty(K); Th = np.empty(K)
    period = ctypes.c_double(); bi = ctypes.c_int32(); ns = ctypes.c_int32()
    sf = np.zeros(L, np.int32); sl = np.zeros(L, np.int32); sp = np.zeros(L, np.int32)
    rc = lib().oracle_literal_solve(L, *ptrs, P, M, beta, n_m, n_v, n_t, K, _ptr(T, ctypes.c_double),
                                    _ptr(Th, ctypes.c_double), ctypes.byref(period), ctypes.byref(bi),
                                    ctypes.byref(ns), _ptr(sf, ctypes.c_int32), _ptr(sl, ctypes.c_int32),
                                    _ptr(sp, ctypes.c_int32))
    if rc < 0:
        raise ValueError("oracle_literal_solve rc=%d" % rc)
    n = ns.value
    return dict(rc=rc, T=T, That=Th, period=period.value, best_iter=bi.value,
                stages=[(int(sf[i]), int(sl[i]), int(sp[i])) for i in range(n)])
