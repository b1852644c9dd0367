#!/usr/bin/env python
"""Benchmark of the MadPipe-DP hot path (BASELINE.json metric: DP cell-updates/s and
time-to-optimal-placement, vs the HBM roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config gpt|batch|...] [--impl ours|reference]

A step is one whole solve of the workload: profile prep,
candidate grid, the DP over every candidate period of this rank's shard, the
MIN all-reduce across ranks, the winner re-solve and its traceback.  For N > 1
the driver launches one process per GPU with torchrun; each rank makes ONE
library call per step (madpipe_solve_dev on a ctx that owns an NCCL
communicator, distributed.context): the library shards the candidates and runs
the all-reduce itself.  torch.distributed is only the process bootstrap and
the timing barrier / max-over-ranks here.

`value` is the whole-job cell-update rate with the chain profile already resident
in HBM (madpipe_solve_dev), timed with CUDA events on the library's stream, max
over ranks.  `e2e` is the same metric through the host-buffer entry
(madpipe_solve on pinned host arrays) with the H2D copies of the inputs and the
D2H read of the result inside the timed region.  `--config batch` times
madpipe_solve_batch over the 512 chains of BASELINE config 5 (host arrays in
both lines: the batch plan is computed on the host).  `--impl reference` times
the CPU oracle (the only reference this tier has) on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "DP cell-updates/s & time-to-optimal-placement at 1/2/4/8 B200 vs HBM roofline"
UNIT = "cell-updates/s"
BYTES_PER_UPDATE = 8          # one fp64 source value per relaxation
L2_FLUSH_BYTES = 256 << 20    # > 126 MB L2


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="gpt")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--force-dist", action="store_true",
                    help="use a ctx with an NCCL communicator (the N-GPU code path) even at N=1")
    return ap.parse_args()


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def is_batch(cfg):
    return "chains" in cfg


def workload(cfg):
    if is_batch(cfg):
        Ls = [c["L"] for c in cfg["chains"]]
        Ps = [c["P"] for c in cfg["chains"]]
        return {"workload": "%s: %d chains (L=%d..%d, P=%d..%d), S=n_delay x n_mem=%dx%d, %d candidate periods "
                            "per chain, per-chain M and beta" % (cfg["name"], len(Ls), min(Ls), max(Ls), min(Ps),
                                                                 max(Ps), cfg["n_delay"], cfg["n_mem"],
                                                                 cfg["n_periods"]),
                "n_chains": len(Ls), "n_delay": cfg["n_delay"], "n_mem": cfg["n_mem"],
                "n_periods": cfg["n_periods"], "v_range": "paper"}
    return {"workload": "%s: L=%d, P=%d, S=n_delay x n_mem=%dx%d, %d candidate periods, M=%.3f GB, "
                        "beta=%.0f GB/s" % (cfg["name"], cfg["L"], cfg["P"], cfg["n_delay"], cfg["n_mem"],
                                            cfg["n_periods"], cfg["M"] / 1e9, cfg["beta"] / 1e9),
            "L": cfg["L"], "P": cfg["P"], "n_delay": cfg["n_delay"], "n_mem": cfg["n_mem"],
            "n_periods": cfg["n_periods"], "M": cfg["M"], "beta": cfg["beta"],
            "v_range": "paper"}


def batch_inputs(cfg):
    import chaingen
    chains, Ps, Ms, Bs = [], [], [], []
    for c in cfg["chains"]:
        ch = chaingen.random_chain(c["seed"])
        assert chaingen.digest(ch) == c["digest"], "generator drift"
        chains.append(ch); Ps.append(c["P"]); Ms.append(c["M"]); Bs.append(c["beta"])
    return chains, Ps, Ms, Bs


def compulsory_bytes(cfg, cands_per_chain=None):
    """a DP table written once and read once, 2 (L+1) P S 8 B per
    candidate (S = n_delay n_mem), summed over every candidate of the workload."""
    S = cfg["n_delay"] * cfg["n_mem"]
    if is_batch(cfg):
        return sum(2 * (c["L"] + 1) * c["P"] * S * 8 * cfg["n_periods"] for c in cfg["chains"])
    return 2 * (cfg["L"] + 1) * cfg["P"] * S * 8 * cfg["n_periods"]


# --------------------------------------------------------------------------- CPU oracle leg
def _offline_seconds(cfg):
    """Per-candidate oracle seconds (1 thread) of the stratified GPT sample in
    configs/gpt_oracle_samples.json (scripts/oracle_gpt_samples.py), linearly
    interpolated over every j; None for other configs."""
    if cfg.get("name") != "gpt":
        return None
    p = os.path.join(ROOT, "configs", "gpt_oracle_samples.json")
    if not os.path.exists(p):
        return None
    import numpy as np
    s = json.load(open(p))["samples"]
    js = np.array([r["j"] for r in s], float)
    ts = np.array([r["oracle_s"] for r in s], float)
    return np.interp(np.arange(cfg["n_periods"]), js, ts)


def oracle_baseline(cfg, one_core=True):
    """The oracle as it stands (SURVEY.md 8(d) 'Oracle timing'), on a
    bounded sample (~10-20 s of CPU work):
      - all cores: candidates j = 0..T-1, one per host thread (T = cores); this round
        contains j* for every config here, so its wall time IS the oracle's early-exit
        time-to-placement on all cores;
      - 1 core: the early-exit scan j = 0..j* single-threaded = the 1-core
        time-to-placement (GPT: 8 candidates);
      - the full sweep on 1 core and on all cores, EXTRAPOLATED from the measured rates
        and the analytic cell-update count of every candidate (not run).
    Returns the cpu_baseline dict and the all-core sample's wall time."""
    import numpy as np

    import chaingen
    import oracle
    T = os.cpu_count() or 1
    if is_batch(cfg):
        chains, Ps, Ms, Bs = batch_inputs(cfg)
        idx = list(range(min(T, len(chains))))
        t0 = time.perf_counter()
        cu = 0
        for i in idx:         # one chain per call, candidates in parallel
            r = oracle.solve(chains[i], Ps[i], Ms[i], Bs[i], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"],
                             early_exit=True, n_threads=T)
            cu += r["cell_updates"]
        dt = time.perf_counter() - t0
        return dict(value=cu / dt, unit=UNIT, cores=T, kind="oracle",
                    sample="batch chains 0..%d solved with early exit (candidates in parallel on %d threads): "
                           "%.3g cell-updates in %.2f s" % (len(idx) - 1, T, cu, dt),
                    time_to_placement_s_per_chain=dt / len(idx)), dt
    ch = chaingen.make(cfg["chain"])
    a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    jstar = cfg["oracle_cand_index"]
    j_hi = min(cfg["n_periods"], max(T, jstar + 1))
    t0 = time.perf_counter()
    r = oracle.solve(ch, *a, j_lo=0, j_hi=j_hi, n_threads=T)
    dt_all = time.perf_counter() - t0
    rate_all = r["cell_updates"] / dt_all
    assert r["cand_index"] == jstar
    out = dict(value=rate_all, unit=UNIT, cores=T, kind="oracle",
               sample="%s candidates j=0..%d (one per thread, full DP tables, incl. winner re-solve + "
                      "traceback): %.3g cell-updates in %.2f s" % (cfg["name"], j_hi - 1, r["cell_updates"], dt_all),
               time_to_placement_allcores_s=dt_all)
    if not one_core:
        return out, dt_all
    t0 = time.perf_counter()
    r1 = oracle.solve(ch, *a, early_exit=True, n_threads=1)
    dt_1 = time.perf_counter() - t0
    assert r1["cand_index"] == jstar
    rate_1 = r1["cell_updates"] / dt_1
    out.update(rate_1core=rate_1,
               rate_1core_sample="early-exit scan j=0..%d on 1 thread: %.3g cell-updates in %.2f s"
                                 % (jstar, r1["cell_updates"], dt_1),
               time_to_placement_1core_s=dt_1)
    import paper_conf_ipps_beaumontes22_b200 as mp
    total = sum(mp.cell_updates(ch, cfg["P"], cfg["n_mem"], cfg["n_delay"], float(t)) for t in r["tau"])
    out["full_sweep_cell_updates"] = total
    off = _offline_seconds(cfg)
    if off is not None:
        sam = json.load(open(os.path.join(ROOT, "configs", "gpt_oracle_samples.json")))["samples"]
        out["stratified_sample_offline"] = {
            "candidates": [r["j"] for r in sam], "cell_updates": sum(r["cell_updates"] for r in sam),
            "oracle_1thread_s": sum(r["oracle_s"] for r in sam),
            "rate_1thread": sum(r["cell_updates"] for r in sam) / sum(r["oracle_s"] for r in sam),
            "what": "SURVEY 8(d) GPT sample (j <= j*, j*+1..8, 16 stratified above, 511/767/1023), each "
                    "candidate's full table by the oracle on 1 thread (8 at a time), scripts/oracle_gpt_samples.py"}
        # the oracle's rate grows with j (longer windows, more skipped transitions), so the
        # full sweep is extrapolated from the stratified per-candidate times measured
        # offline, rescaled to this host by the live 1-core scan of j = 0..j*
        f = dt_1 / float(off[:jstar + 1].sum())
        one = f * float(off.sum())
        out.update(full_sweep_1core_s_extrapolated=one,
                   full_sweep_allcores_s_extrapolated=one * rate_1 / rate_all,
                   extrapolation="NOT RUN: sum over all %d candidates of the per-candidate 1-thread oracle "
                                 "times of configs/gpt_oracle_samples.json (34 stratified candidates, "
                                 "interpolated in j), x %.3f = this host's live 1-thread time for j=0..%d / "
                                 "the offline one; all cores = that / (all-core rate / 1-core rate)"
                                 % (cfg["n_periods"], f, jstar))
    else:
        out.update(full_sweep_1core_s_extrapolated=total / rate_1,
                   full_sweep_allcores_s_extrapolated=total / rate_all,
                   extrapolation="NOT RUN: analytic cell-updates of all %d candidates / measured rates"
                                 % cfg["n_periods"])
    return out, dt_all


def run_reference(args, cfg):
    rank, world, _ = env_rank()
    if rank != 0:
        return
    for _ in range(args.warmup):
        oracle_baseline(cfg, one_core=False)
    vals, times = [], []
    cpu = None
    for i in range(args.steps):
        # the 1-core scan (~20 s at GPT) only once, on the last step
        cpu, dt = oracle_baseline(cfg, one_core=(i == args.steps - 1))
        vals.append(cpu["value"]); times.append(dt)
    v = statistics.median(vals)
    cpu["value"] = v
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.median(times),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (chaingen, seeded)", "config": workload(cfg), "cpu_baseline": cpu,
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------- clocks
class ClockSampler:
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None
        self.lines = []

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q,
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.p = None
        return self

    def _read(self):
        for ln in self.p.stdout:
            self.lines.append(ln.strip())

    def __exit__(self, *a):
        if self.p:
            self.p.terminate()
            try:
                self.p.wait(2)
            except Exception:
                self.p.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[0])); mx.append(float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def _profile_json(name):
    p = os.path.join(ROOT, "profiles", name)
    return json.load(open(p)) if os.path.exists(p) else None


# --------------------------------------------------------------------------- GPU leg
def main():
    args = parse()
    from paper_conf_ipps_beaumontes22_b200 import configs
    cfg = configs.load(args.config)
    if args.impl == "reference":
        run_reference(args, cfg)
        return
    import numpy as np
    import torch
    import torch.distributed as dist

    import chaingen
    import paper_conf_ipps_beaumontes22_b200 as mp
    from paper_conf_ipps_beaumontes22_b200 import distributed

    rank, world, local = env_rank()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    use_dist = world > 1 or args.force_dist
    stream = torch.cuda.current_stream(dev)
    if use_dist:
        if os.environ.get("NCCL_DEBUG", "VERSION").upper() in ("VERSION", "WARN"):
            os.environ["NCCL_DEBUG"] = "NONE"      # keep stdout to the one JSON line (VERSION and WARN
            #                                        both print "NCCL version ..." to stdout at init)
        dist.init_process_group("nccl", device_id=dev)
        ctx = distributed.context(local, stream=stream.cuda_stream)   # ctx-owned NCCL communicator
    else:
        ctx = mp.Context(local, stream=stream.cuda_stream)
    ctx.set_timing(True)

    batch = is_batch(cfg)
    d = (cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    if batch:
        chains, Ps, Ms, Bs = batch_inputs(cfg)
        dchain = pinned = None
    else:
        ch = chaingen.make(cfg["chain"])
        assert chaingen.digest(ch) == cfg["digest"], "generator drift"
        a = (cfg["P"], cfg["M"], cfg["beta"]) + d
        dchain = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).to(dev) for k in ("uF", "uB", "W", "a")}
        pinned = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).pin_memory().numpy()
                  for k in ("uF", "uB", "W", "a")}
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)

    def step(chain, early_exit=False):
        """One solve = one library call; returns (winner summary, this rank's counts)."""
        if batch:
            res = ctx.solve_batch(chains, Ps, Ms, Bs, *d, early_exit=early_exit)
            summ = {"feasible": sum(r["cand_index"] >= 0 for r in res),
                    "cand_index_sum": sum(r["cand_index"] for r in res)}
            cu = sum(r["cell_updates"] for r in res)
        else:
            res = ctx.solve_dev(chain, *a, early_exit=early_exit) if chain is dchain else \
                ctx.solve(chain, *a, early_exit=early_exit)
            summ = {"cand_index": res["cand_index"], "period": res["period"],
                    "special_load": res["special_load"], "n_stages": len(res["stages"])}
            cu = res["cell_updates"]
        t = ctx.last_timing()
        cnt = ctx.last_counts()
        sb = ctx.last_step_bytes()
        return summ, dict(cu=cu, eff=cnt["effective_updates"], useful=cnt["useful_updates"],
                          moved=sb["load_bytes"] + sb["store_bytes"], launches=t["launches"], kern_ms=t["step_ms"])

    def timed(chain, k, early_exit=False):
        dev_ms, wall, cnts = [], [], []
        io = (0, 0)
        summ = None
        for _ in range(k):
            flush.zero_()
            torch.cuda.synchronize(dev)
            if use_dist:
                dist.barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            w0 = time.perf_counter()
            summ, c = step(chain, early_exit)
            w1 = time.perf_counter()
            e1.record(stream)
            torch.cuda.synchronize(dev)
            dev_ms.append(e0.elapsed_time(e1))
            wall.append(w1 - w0)
            cnts.append(c)
            last_io = ctx.last_io()
            io = (last_io["h2d_bytes"], last_io["d2h_bytes"])
        return dict(summ=summ, dev_ms=dev_ms, wall=wall, cnts=cnts, io=io)

    main_chain = pinned if batch else dchain
    for _ in range(args.warmup):
        step(main_chain)
    torch.cuda.synchronize(dev)
    with ClockSampler(local) as clk:
        main_run = timed(main_chain, args.steps)
    e2e_run = None if args.no_e2e else timed(pinned, args.steps)
    ee_run = timed(main_chain, args.steps, early_exit=True)

    def reduce(x, op):
        if not use_dist:
            return x
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=op)
        return t.item()

    SUM, MAX = (dist.ReduceOp.SUM, dist.ReduceOp.MAX) if use_dist else (None, None)
    K = args.steps
    last = main_run["cnts"][-1]
    tot_ms = reduce(sum(main_run["dev_ms"]), MAX)
    cu_step = reduce(last["cu"], SUM)
    eff_step = reduce(last["eff"], SUM)
    useful_step = reduce(last["useful"], SUM)
    value = cu_step * K / (tot_ms / 1e3)
    kern_ms = reduce(sum(c["kern_ms"] for c in main_run["cnts"]), MAX)     # the dominant kernel, max rank
    launches = int(reduce(sum(c["launches"] for c in main_run["cnts"]), SUM))
    ttp = reduce(statistics.median(main_run["wall"]), MAX)
    ttp_ee = reduce(statistics.median(ee_run["wall"]), MAX)
    moved_step = reduce(last["moved"], SUM) / world          # per GPU
    e2e = None
    if e2e_run:
        e2e_ms = reduce(sum(e2e_run["dev_ms"]), MAX)
        e2e_wall = reduce(sum(e2e_run["wall"]), MAX)
        e2e = {"value": cu_step * K / (max(e2e_ms, 1e3 * e2e_wall) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(reduce(e2e_run["io"][0], SUM)),
               "d2h_bytes_per_step": int(reduce(e2e_run["io"][1], SUM)),
               "ms_per_step": max(e2e_ms, 1e3 * e2e_wall) / K,
               "entry": ("madpipe_solve_batch" if batch else "madpipe_solve") + " on pinned host arrays"
                        + (" (ctx with an NCCL communicator of %d ranks)" % world if use_dist else "")}
    if rank != 0:
        if use_dist:
            dist.destroy_process_group()
        return
    peaks = _profile_json("../MEASURED_PEAKS.json") or {}
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    # roofline of the dominant kernel: SURVEY.md 8(d)'s compulsory bytes --
    # every candidate's table written once and read once -- over the kernel's own time
    comp_step = compulsory_bytes(cfg) / world
    achieved = comp_step * K / (kern_ms / 1e3) / 1e9 if kern_ms > 0 else None
    moved_rate = moved_step * K / (kern_ms / 1e3) / 1e9 if kern_ms > 0 and moved_step > 0 else None
    units = useful_step if useful_step > 0 else eff_step
    streaming = units / world * K * BYTES_PER_UPDATE / (kern_ms / 1e3) / 1e9 if kern_ms > 0 else None
    traffic = _profile_json("r02b_step_traffic.json") if args.config == "gpt" else None
    pipes = _profile_json("r02b_step_pipes.json") if args.config == "gpt" else None
    fp64 = _profile_json("r02_fp64_peak.json")
    n_launch = (cfg["L"] + 1) // 2 if not batch else None
    roof = {"bound": "hbm", "kernel": ctx.last_kernel(), "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
            "frac": (achieved / hbm_peak) if achieved else None,
            "traffic": (traffic["dram_bytes_per_solve"] / traffic["step_launches_per_solve"]) if traffic else None,
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured copy bandwidth)",
            "algorithmic_bytes": "compulsory (SURVEY.md 8(d)): 2 (L+1) P n_delay n_mem 8 B per candidate = "
                                 "%.4g B per step per GPU" % comp_step,
            "algorithmic_bytes_per_launch": comp_step / n_launch if n_launch else None,
            "kernel_ms_per_step": kern_ms / K,
            "kernel_share": kern_ms / tot_ms if tot_ms else None,
            "moved_bytes_per_step": moved_step,
            "moved_bytes_rate_gbs": moved_rate,
            "moved_bytes_efficiency": (moved_rate / hbm_peak) if moved_rate else None,
            "moved_bytes": "source-row segments loaded + output rows stored by the step kernel (DESIGN.md 6.1)",
            "streaming_equiv": streaming,
            "streaming_equiv_units": "%d B x %s / step-kernel time" % (
                BYTES_PER_UPDATE, "useful relaxations" if useful_step > 0 else "effective relaxations")}
    if traffic:
        roof["traffic_source"] = traffic.get("source")
        roof["traffic_over_moved"] = traffic["dram_bytes_per_solve"] / traffic["moved_bytes_per_solve"]
        roof["traffic_over_compulsory"] = traffic["dram_bytes_per_solve"] / traffic["compulsory_bytes_per_solve"]
    if pipes:
        roof.update({k: pipes[k] for k in ("fp64_pct", "alu_pct", "issue_pct", "warps_active_pct", "dram_pct",
                                           "lsu_pct") if k in pipes})
        roof["pipes_source"] = pipes.get("source")
    if fp64:
        roof["fp64_peak_dadd_per_s"] = fp64.get("dadd_per_s")
    cpu = None
    if world == 1 and not args.no_cpu:
        cpu, _ = oracle_baseline(cfg)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": tot_ms / K, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic (chaingen, seeded)",
        "config": {**workload(cfg),
                   "parallelism": ("candidates %s over %d rank(s); one library call per rank and step, "
                                   "NCCL all-reduce(MIN) inside the library" % (
                                       "LPT-planned" if batch else "interleaved", world)) if use_dist
                   else "1 GPU, %s" % ("madpipe_solve_batch (host arrays)" if batch else "madpipe_solve_dev"),
                   "l2": "DP tables >> L2 and a %d MB L2 flush between steps" % (L2_FLUSH_BYTES >> 20)},
        "time_to_placement_s": ttp, "time_to_placement_early_exit_s": ttp_ee,
        "cell_updates_per_step": cu_step,
        "effective_updates_per_step": eff_step,
        "effective_updates_per_s": eff_step * K / (tot_ms / 1e3),
        "useful_updates_per_step": useful_step,
        "result": dict(main_run["summ"], **(
            {"oracle_cand_index_sum": sum(c["oracle_cand_index"] for c in cfg["chains"]),
             "matches_oracle": main_run["summ"]["cand_index_sum"] == sum(c["oracle_cand_index"] for c in cfg["chains"])}
            if batch else {"oracle_cand_index": cfg.get("oracle_cand_index"),
                           "matches_oracle": main_run["summ"]["cand_index"] == cfg.get("oracle_cand_index")})),
        "roofline": roof,
        "e2e": e2e, "gpu_launches": launches, "clocks": clk.summary(), "cpu_baseline": cpu,
    }
    print(json.dumps(line), flush=True)
    if use_dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
