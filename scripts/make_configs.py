"""Write configs/*.json: the five BASELINE.json workloads.

Calls only chaingen (profiles) and oracle/ (M_free, feasibility): every stored
value is either a recipe constant or written by this script from the oracle.

M_free = the largest per-GPU model memory of the oracle's solution at
M = 2^62 (normal GPU: M(k,l,g_s); special GPU: sum M(k,l,g_s - 1), with the
exact 1F1B* groups g_s of the simulator).  "Tight" M = factor * M_free; if no
candidate is feasible the factor is raised by 0.05 until one is.
"""
from __future__ import annotations

import json
import math
import os
import sys
import time
from concurrent.futures import ProcessPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import chaingen  # noqa: E402
import oracle  # noqa: E402
from oracle import simulator  # noqa: E402

OUT = os.path.join(ROOT, "configs")
BIG = 2 ** 62
GB = 1e9


def m_free(ch, P, beta, n_m, n_v, n_c, threads):
    r = oracle.solve(ch, P, BIG, beta, n_m, n_v, n_c, early_exit=True, n_threads=threads)
    if r["rc"] != 0:
        raise RuntimeError("infeasible even at M=2^62")
    rep = simulator.check_allocation(ch, P, BIG, beta, r["period"], r["stages"], build_pattern=False)
    mf = max(rep["normal_mem"] + [rep["special_mem_model"]])
    return int(mf), r


def tighten(ch, P, beta, n_m, n_v, n_c, factor, threads, mf, assert_binding=False, free_r=None):
    f = factor
    while True:
        M = int(f * mf)
        r = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, early_exit=True, n_threads=threads)
        if r["rc"] == 0:
            break
        f = round(f + 0.05, 2)
    if assert_binding and free_r is not None:
        rep = simulator.check_allocation(ch, P, M, beta, free_r["period"], free_r["stages"],
                                         build_pattern=False)
        if not any("needs" in e or "model memory" in e for e in rep["errors"]):
            raise RuntimeError("M is not binding: the M=inf solution fits")
    return M, f, r


def single(name, chain_spec, P, beta, n_m, n_v, n_c, factor=None, M_fixed=None, threads=8,
           assert_binding=False, note=""):
    t0 = time.time()
    ch = chaingen.make(chain_spec)
    mf, fr = m_free(ch, P, beta, n_m, n_v, n_c, threads)
    if M_fixed is not None:
        M, f = int(M_fixed), None
        r = oracle.solve(ch, P, M, beta, n_m, n_v, n_c, early_exit=True, n_threads=threads)
        assert r["rc"] == 0, "fixed M infeasible"
    else:
        M, f, r = tighten(ch, P, beta, n_m, n_v, n_c, factor, threads, mf, assert_binding, fr)
    cfg = dict(name=name, chain=chain_spec, L=len(ch["uF"]), P=P, M=M, beta=beta, n_mem=n_m,
               n_delay=n_v, n_periods=n_c, v_range=0, mem_factor=f, M_free=mf,
               M_free_cand=fr["cand_index"], oracle_cand_index=r["cand_index"],
               digest=chaingen.digest(ch), note=note)
    with open(os.path.join(OUT, name + ".json"), "w") as fh:
        json.dump(cfg, fh, indent=1)
    print("%-14s L=%d P=%d M=%.3f GB (M_free %.3f GB, factor %s) j*=%d  %.1fs" % (
        name, cfg["L"], P, M / GB, mf / GB, f, r["cand_index"], time.time() - t0), flush=True)
    return cfg


def _batch_one(seed):
    ch = chaingen.random_chain(seed)
    P, beta, mfac = chaingen.random_batch_params(seed)
    mf, fr = m_free(ch, P, beta, 8, 32, 64, 1)
    M, f, r = tighten(ch, P, beta, 8, 32, 64, mfac, 1, mf)
    return dict(seed=seed, L=len(ch["uF"]), P=P, beta=beta, M=M, M_free=mf, mem_factor=f,
                oracle_cand_index=r["cand_index"], digest=chaingen.digest(ch))


def batch(n=512, first_seed=1000, workers=8):
    t0 = time.time()
    with ProcessPoolExecutor(workers) as ex:
        chains = list(ex.map(_batch_one, range(first_seed, first_seed + n)))
    cfg = dict(name="batch", n_chains=n, n_mem=8, n_delay=32, n_periods=64, v_range=0,
               chains=chains)
    with open(os.path.join(OUT, "batch.json"), "w") as fh:
        json.dump(cfg, fh, indent=1)
    print("batch: %d chains in %.1fs" % (n, time.time() - t0))


if __name__ == "__main__":
    os.makedirs(OUT, exist_ok=True)
    which = sys.argv[1:] or ["toy", "resnet50", "inception_v3", "vgg19", "gpt", "batch"]
    oracle.build()
    if "toy" in which:
        single("toy", {"family": "toy", "seed": 1}, 2, 12 * GB, 4, 4, 32, factor=0.6)
    if "resnet50" in which:
        single("resnet50", {"family": "resnet50", "seed": 2}, 8, 12 * GB, 8, 32, 1024,
               M_fixed=6 * GB)
    if "inception_v3" in which:
        single("inception_v3", {"family": "inception_v3", "seed": 3}, 16, 12 * GB, 8, 128, 1024,
               factor=0.6, assert_binding=True)
    if "vgg19" in which:
        single("vgg19", {"family": "vgg19", "seed": 4}, 16, 12 * GB, 8, 128, 1024, factor=0.6,
               assert_binding=True)
    if "gpt" in which:
        single("gpt", {"family": "gpt", "seed": 5}, 64, 12 * GB, 8, 512, 1024, factor=0.6)
    if "batch" in which:
        batch()
