"""B200-native MadPipe-DP hot path (Beaumont, Eyraud-Dubois, Shilova, hal-03025305).

Thin Python layer over the C ABI of ``libmadpipe.so`` (include/madpipe.h): the
memory-aware dynamic program of MadPipe section 4.2 evaluated over a batched
sweep of candidate periods (replacing Algorithm 1's serial search),
with a device-side traceback.  PyTorch is used only for device memory, streams
and process groups (see ``distributed.py``).  There is no CPU fallback.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _native as N
from ._native import VRANGE_PAPER, VRANGE_SAFE, MadpipeError  # noqa: F401

__all__ = ["Context", "validate", "shard", "cell_updates", "schedule", "get_unique_id", "batch_plan",
           "resolve_plan", "VRANGE_PAPER", "VRANGE_SAFE", "MadpipeError"]


def get_unique_id() -> bytes:
    """madpipe_get_unique_id: the 128-byte NCCL id one rank creates for the others."""
    b = ctypes.create_string_buffer(128)
    N.check(N.lib().madpipe_get_unique_id(b))
    return b.raw


class _Batch:
    """Keeps the ctypes arrays of a batch of host chains alive for one call."""

    def __init__(self, chains, Ps, Ms, betas):
        self.hcs = [N.HostChain(c) for c in chains]
        self.n = len(self.hcs)
        self.arr = (N.Chain * self.n)(*[h.c for h in self.hcs])
        self.P = np.ascontiguousarray(Ps, np.int32)
        self.M = np.ascontiguousarray(Ms if Ms is not None else np.ones(self.n), np.int64)
        self.B = np.ascontiguousarray(betas, np.float64)

    def args(self):
        return (self.n, self.arr, self.P.ctypes.data_as(N._i32p), self.M.ctypes.data_as(N._i64p),
                self.B.ctypes.data_as(N._dp))


def batch_plan(chains, Ps, betas, n_mem, n_delay, n_periods, world):
    """madpipe_batch_plan (host only): (owner[n][n_periods], load[world], cost[n][n_periods])."""
    b = _Batch(chains, Ps, None, betas)
    d = N.make_disc(n_mem, n_delay, n_periods)
    owner = np.empty((b.n, n_periods), np.int32)
    load = np.empty(world, np.int64)
    cost = np.empty((b.n, n_periods), np.int64)
    N.check(N.lib().madpipe_batch_plan(b.n, b.arr, b.P.ctypes.data_as(N._i32p), b.B.ctypes.data_as(N._dp),
                                       ctypes.byref(d), int(world), owner.ctypes.data_as(N._i32p),
                                       load.ctypes.data_as(N._i64p), cost.ctypes.data_as(N._i64p)))
    return owner, load, cost


def resolve_plan(chains, Ps, betas, n_mem, n_delay, n_periods, j_star, world):
    """madpipe_resolve_plan (host only): the rank re-solving each chain's winner (-1: none)."""
    b = _Batch(chains, Ps, None, betas)
    d = N.make_disc(n_mem, n_delay, n_periods)
    js = np.ascontiguousarray(j_star, np.int32)
    owner = np.empty(b.n, np.int32)
    N.check(N.lib().madpipe_resolve_plan(b.n, b.arr, b.P.ctypes.data_as(N._i32p), b.B.ctypes.data_as(N._dp),
                                         ctypes.byref(d), js.ctypes.data_as(N._i32p), int(world),
                                         owner.ctypes.data_as(N._i32p)))
    return owner


def validate(chain, P, M, beta, n_mem, n_delay, n_periods, v_range=VRANGE_PAPER) -> int:
    """madpipe_validate (host only): 0 or -1 (EINVAL)."""
    hc = N.HostChain(chain)
    d = N.make_disc(n_mem, n_delay, n_periods, v_range)
    return N.lib().madpipe_validate(ctypes.byref(hc.c), int(P), int(M), float(beta), ctypes.byref(d))


def shard(n_periods, rank, world):
    """madpipe_shard (host only): the candidate indices owned by a rank."""
    out = np.zeros(max(1, n_periods), np.int32)
    cnt = ctypes.c_int32()
    N.check(N.lib().madpipe_shard(n_periods, rank, world, out.ctypes.data_as(N._i32p), ctypes.byref(cnt)))
    return [int(x) for x in out[:cnt.value]]


def cell_updates(chain, P, n_mem, n_delay, tau) -> int:
    hc = N.HostChain(chain)
    d = N.make_disc(n_mem, n_delay, 1)
    return int(N.lib().madpipe_cell_updates(ctypes.byref(hc.c), int(P), ctypes.byref(d), float(tau)))


def schedule(chain, beta, period, stages):
    """madpipe_schedule (host only): the 1F1B* pattern of a contiguous allocation
    (P:101-113).  ``stages`` = [(first, last, ...), ...] in chain order.
    Returns a list of dicts (kind 'stage'/'comm', stage, group, F=(start, shift),
    B=(start, shift), f_len, b_len), or None if an item exceeds the period."""
    hc = N.HostChain(chain)
    first = np.ascontiguousarray([s[0] for s in stages], np.int32)
    last = np.ascontiguousarray([s[1] for s in stages], np.int32)
    ops = (N.Op * (2 * len(stages) - 1))()
    n = ctypes.c_int32()
    rc = N.lib().madpipe_schedule(ctypes.byref(hc.c), float(beta), float(period), len(stages),
                                  first.ctypes.data_as(N._i32p), last.ctypes.data_as(N._i32p), ops,
                                  ctypes.byref(n))
    if rc == N.INFEASIBLE:
        return None
    N.check(rc)
    return [dict(kind="comm" if o.kind else "stage", stage=o.stage, group=o.group,
                 F=(o.f_start, o.f_shift), B=(o.b_start, o.b_shift), f_len=o.f_len, b_len=o.b_len)
            for o in ops[:n.value]]


class _DevChain:
    def __init__(self, d):
        self.L = int(d["uF"].numel())
        self.keep = d
        self.c = N.Chain(self.L, d["uF"].data_ptr(), d["uB"].data_ptr(), d["W"].data_ptr(),
                         d["a"].data_ptr())


def _any_chain(chain):
    if hasattr(chain["uF"], "is_cuda") and chain["uF"].is_cuda:
        return _DevChain(chain)
    return N.HostChain(chain)


class Context:
    """A libmadpipe context bound to one CUDA device (madpipe_ctx_create): rank ``rank`` of
    ``world``; with ``nccl_id`` (128 bytes, see distributed.context) the ctx owns the NCCL
    communicator its solves all-reduce over."""

    def __init__(self, device: int = 0, stream=None, mem_budget: int = 0, rank: int = 0, world: int = 1,
                 nccl_id: bytes | None = None):
        self._lib = N.lib()
        h = ctypes.c_void_p()
        rc = self._lib.madpipe_ctx_create(ctypes.byref(h), int(device), int(rank), int(world),
                                          nccl_id, ctypes.c_void_p(stream) if stream else None,
                                          int(mem_budget))
        if rc != N.OK:
            raise MadpipeError(rc, N.last_error(None))
        self.h = h
        self.device = device
        self.rank, self.world = int(rank), int(world)

    def info(self):
        r = ctypes.c_int32(); w = ctypes.c_int32(); v = ctypes.c_int32()
        N.check(self._lib.madpipe_ctx_info(self.h, ctypes.byref(r), ctypes.byref(w), ctypes.byref(v)))
        return dict(rank=r.value, world=w.value, nccl_version=v.value)

    def close(self):
        if getattr(self, "h", None):
            self._lib.madpipe_ctx_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ------------------------------------------------------------------ hot path
    def solve(self, chain, P, M, beta, n_mem, n_delay, n_periods, v_range=VRANGE_PAPER,
              early_exit=False):
        hc = N.HostChain(chain)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range, early_exit)
        buf = N.AllocBuf(hc.L)
        rc = self._lib.madpipe_solve(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta),
                                     ctypes.byref(d), ctypes.byref(buf.s))
        N.check(rc, self.h)
        return buf.result(rc)

    def solve_dev(self, dchain, P, M, beta, n_mem, n_delay, n_periods, v_range=VRANGE_PAPER,
                  early_exit=False):
        """``dchain``: dict of CUDA tensors uF, uB (float64), W, a (int64) on this device."""
        L = int(dchain["uF"].numel())
        c = N.Chain(L, dchain["uF"].data_ptr(), dchain["uB"].data_ptr(), dchain["W"].data_ptr(),
                    dchain["a"].data_ptr())
        d = N.make_disc(n_mem, n_delay, n_periods, v_range, early_exit)
        buf = N.AllocBuf(L)
        rc = self._lib.madpipe_solve_dev(self.h, ctypes.byref(c), int(P), int(M), float(beta),
                                         ctypes.byref(d), ctypes.byref(buf.s))
        N.check(rc, self.h)
        return buf.result(rc)

    def sweep(self, chain, P, M, beta, n_mem, n_delay, n_periods, rank, world, j_local_ptr,
              v_range=VRANGE_PAPER, early_exit=False) -> int:
        """Evaluate this rank's candidates; writes the local minimum feasible index
        (INT32_MAX if none) to the int32 device buffer at ``j_local_ptr``.  ``chain``
        is a host dict of arrays or a dict of CUDA tensors."""
        hc = _any_chain(chain)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range, early_exit)
        cu = ctypes.c_int64()
        N.check(self._lib.madpipe_sweep(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta),
                                        ctypes.byref(d), int(rank), int(world),
                                        ctypes.c_void_p(j_local_ptr), ctypes.byref(cu)), self.h)
        return cu.value

    def resolve(self, chain, P, M, beta, n_mem, n_delay, n_periods, j_star_ptr,
                v_range=VRANGE_PAPER):
        hc = _any_chain(chain)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range)
        buf = N.AllocBuf(hc.L)
        rc = self._lib.madpipe_resolve(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta),
                                       ctypes.byref(d), ctypes.c_void_p(j_star_ptr), ctypes.byref(buf.s))
        N.check(rc, self.h)
        return buf.result(rc)

    def solve_batch(self, chains, Ps, Ms, betas, n_mem, n_delay, n_periods, v_range=VRANGE_PAPER,
                    early_exit=False):
        b = _Batch(chains, Ps, Ms, betas)
        bufs = [N.AllocBuf(h.L) for h in b.hcs]
        outs = (N.Alloc * b.n)(*[x.s for x in bufs])
        d = N.make_disc(n_mem, n_delay, n_periods, v_range, early_exit)
        N.check(self._lib.madpipe_solve_batch(self.h, *b.args(), ctypes.byref(d), outs), self.h)
        return self._batch_results(bufs, outs)

    @staticmethod
    def _batch_results(bufs, outs):
        res = []
        for x, o in zip(bufs, outs):
            x.s = o
            res.append(x.result(N.OK if o.cand_index >= 0 else N.INFEASIBLE))
        return res

    def sweep_batch(self, chains, Ps, Ms, betas, n_mem, n_delay, n_periods, rank, world, v_range=VRANGE_PAPER,
                    early_exit=False):
        """madpipe_sweep_batch: (j_local[n], cell_updates[n]) of rank ``rank`` of ``world``."""
        b = _Batch(chains, Ps, Ms, betas)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range, early_exit)
        jl = np.empty(b.n, np.int32)
        cu = np.empty(b.n, np.int64)
        N.check(self._lib.madpipe_sweep_batch(self.h, *b.args(), ctypes.byref(d), int(rank), int(world),
                                              jl.ctypes.data_as(N._i32p), cu.ctypes.data_as(N._i64p)), self.h)
        return jl, cu

    def resolve_batch(self, chains, Ps, Ms, betas, n_mem, n_delay, n_periods, j_star, rank, world,
                      v_range=VRANGE_PAPER):
        """madpipe_resolve_batch: results of the winners rank ``rank`` owns ({chain: result})."""
        b = _Batch(chains, Ps, Ms, betas)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range)
        js = np.ascontiguousarray(j_star, np.int32)
        bufs = [N.AllocBuf(h.L) for h in b.hcs]
        for x in bufs:
            x.s.cand_index = -2                      # marks "not written by this rank"
        outs = (N.Alloc * b.n)(*[x.s for x in bufs])
        N.check(self._lib.madpipe_resolve_batch(self.h, *b.args(), ctypes.byref(d), js.ctypes.data_as(N._i32p),
                                                int(rank), int(world), outs), self.h)
        res = {}
        for i, (x, o) in enumerate(zip(bufs, outs)):
            if o.cand_index != -2:
                x.s = o
                res[i] = x.result(N.OK if o.cand_index >= 0 else N.INFEASIBLE)
        return res

    # ------------------------------------------------------------------ parity exports
    def candidates(self, chain, P, M, beta, n_mem, n_delay, n_periods, v_range=VRANGE_PAPER):
        hc = N.HostChain(chain)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range)
        tau = np.empty(n_periods)
        root = np.empty(n_periods)
        N.check(self._lib.madpipe_candidates(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta),
                                             ctypes.byref(d), tau.ctypes.data_as(N._dp),
                                             root.ctypes.data_as(N._dp)), self.h)
        return tau, root

    def dp_table(self, chain, P, M, beta, n_mem, n_delay, n_periods, j, v_range=VRANGE_PAPER,
                 with_arg=True):
        hc = N.HostChain(chain)
        d = N.make_disc(n_mem, n_delay, n_periods, v_range)
        A = np.empty((hc.L + 1, P, n_delay, n_mem), np.float64)
        ARG = np.empty((hc.L + 1, P, n_delay, n_mem), np.int32) if with_arg else None
        N.check(self._lib.madpipe_dp_table(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta),
                                           ctypes.byref(d), int(j), A.ctypes.data_as(N._dp),
                                           ARG.ctypes.data_as(N._i32p) if with_arg else None),
                self.h)
        return A, ARG

    # ------------------------------------------------------------------ NEXT row f1
    def solve_paper(self, chain, P, M, beta, n_mem=11, n_delay=51, n_tp=101, K=10):
        """Paper-literal MadPipe-DP + Algorithm 1 (P:173-205, P:233 discretisation)."""
        hc = N.HostChain(chain)
        buf = N.AllocBuf(hc.L)
        T = np.empty(K); Th = np.empty(K)
        rc = self._lib.madpipe_solve_paper(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta), int(n_mem),
                                           int(n_delay), int(n_tp), int(K), ctypes.byref(buf.s),
                                           T.ctypes.data_as(N._dp), Th.ctypes.data_as(N._dp))
        N.check(rc, self.h)
        r = buf.result(rc)
        r.update(T=T, That=Th, best_iter=r["cand_index"])
        return r

    def literal_table(self, chain, P, M, beta, n_mem, n_delay, n_tp, That, with_arg=True):
        hc = N.HostChain(chain)
        A = np.empty((hc.L + 1, P, n_tp, n_delay, n_mem), np.float64)
        ARG = np.empty(A.shape, np.int32) if with_arg else None
        N.check(self._lib.madpipe_literal_table(self.h, ctypes.byref(hc.c), int(P), int(M), float(beta),
                                                int(n_mem), int(n_delay), int(n_tp), float(That),
                                                A.ctypes.data_as(N._dp),
                                                ARG.ctypes.data_as(N._i32p) if with_arg else None), self.h)
        return A, ARG

    def set_timing(self, per_launch: bool):
        N.check(self._lib.madpipe_set_timing(self.h, 1 if per_launch else 0), self.h)

    def last_io(self):
        a = ctypes.c_int64(); b = ctypes.c_int64()
        N.check(self._lib.madpipe_last_io(self.h, ctypes.byref(a), ctypes.byref(b)))
        return dict(h2d_bytes=a.value, d2h_bytes=b.value)

    def last_counts(self):
        a = ctypes.c_int64(); b = ctypes.c_int64(); c = ctypes.c_int64()
        N.check(self._lib.madpipe_last_counts(self.h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)))
        return dict(cell_updates=a.value, effective_updates=b.value, useful_updates=c.value)

    def last_step_bytes(self):
        """Algorithmic bytes of the step kernel in the last sweep (madpipe_last_step_bytes)."""
        a = ctypes.c_int64(); b = ctypes.c_int64(); c = ctypes.c_int64()
        N.check(self._lib.madpipe_last_step_bytes(self.h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)))
        return dict(load_bytes=a.value, store_bytes=b.value, segments=c.value)

    def last_kernel(self):
        """Step kernel of the largest batch of the last sweep (madpipe_last_kernel)."""
        k = ctypes.c_int32()
        N.check(self._lib.madpipe_last_kernel(self.h, ctypes.byref(k)))
        return {0: "step_kernel", 2: "step_persist_kernel",
                3: "pair_step_kernel"}.get(k.value, None)

    def last_timing(self):
        s = ctypes.c_double(); k = ctypes.c_double(); n = ctypes.c_int64()
        N.check(self._lib.madpipe_last_timing(self.h, ctypes.byref(s), ctypes.byref(k), ctypes.byref(n)))
        return dict(sweep_ms=s.value, step_ms=k.value, launches=n.value)
