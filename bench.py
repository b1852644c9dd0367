#!/usr/bin/env python
"""Benchmark of the MadPipe-DP hot path (BASELINE.json metric: DP cell-updates/s and
time-to-optimal-placement, vs the HBM roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config gpt] [--impl ours|reference]

A step is one whole solve of the workload: profile prep,
candidate grid, the DP over every candidate period of this rank's shard, the
min-reduction across ranks, the winner re-solve and its traceback.  For N > 1 the
driver launches one process per GPU with torchrun; candidates are sharded over
the ranks and min-reduced with one NCCL all-reduce.

`value` is the whole-job cell-update rate with the chain profile already resident
in HBM (madpipe_solve_dev / madpipe_sweep on device arrays), timed with CUDA events
on the library's stream, max over ranks.  `e2e` is the same metric through the
host-buffer entry (madpipe_solve / madpipe_sweep on pinned host arrays) with the
H2D copies of the inputs and the D2H read of the result inside the timed region.
`--impl reference` times the CPU oracle (the only reference this tier has) on a
bounded sample of the same workload.
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
                    help="use the multi-GPU controller (sweep + NCCL all-reduce + resolve) even at N=1")
    return ap.parse_args()


def env_rank():
    return (int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)),
            int(os.environ.get("LOCAL_RANK", 0)))


def workload(cfg):
    return {"workload": "%s: L=%d, P=%d, S=n_delay x n_mem=%dx%d, %d candidate periods, M=%.3f GB, "
                        "beta=%.0f GB/s" % (cfg["name"], cfg["L"], cfg["P"], cfg["n_delay"], cfg["n_mem"],
                                            cfg["n_periods"], cfg["M"] / 1e9, cfg["beta"] / 1e9),
            "L": cfg["L"], "P": cfg["P"], "n_delay": cfg["n_delay"], "n_mem": cfg["n_mem"],
            "n_periods": cfg["n_periods"], "M": cfg["M"], "beta": cfg["beta"],
            "v_range": "paper"}


# --------------------------------------------------------------------------- CPU oracle leg
def oracle_sample(cfg, threads=None):
    """The oracle as it stands on a bounded sample of the workload: the first T
    candidate periods (one per host thread), full DP tables, no early exit."""
    import chaingen
    import oracle
    T = threads or os.cpu_count() or 1
    ch = chaingen.make(cfg["chain"])
    j_hi = min(cfg["n_periods"], T)
    t0 = time.perf_counter()
    r = oracle.solve(ch, cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"],
                     cfg["n_periods"], j_lo=0, j_hi=j_hi, n_threads=T)
    dt = time.perf_counter() - t0
    return dict(value=r["cell_updates"] / dt, unit=UNIT, cores=T, kind="oracle",
                sample="%s candidates j=0..%d (one per thread), full DP tables, %.3g cell-updates "
                       "in %.2f s (incl. winner re-solve + traceback)" % (cfg["name"], j_hi - 1,
                                                                         r["cell_updates"], dt)), dt


def run_reference(args, cfg):
    rank, world, _ = env_rank()
    if rank != 0:
        return
    for _ in range(args.warmup):
        oracle_sample(cfg)
    vals, times = [], []
    cpu = None
    for _ in range(args.steps):
        cpu, dt = oracle_sample(cfg)
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
    from paper_conf_ipps_beaumontes22_b200.distributed import solve_distributed

    rank, world, local = env_rank()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    use_dist = world > 1 or args.force_dist
    if use_dist:
        if os.environ.get("NCCL_DEBUG", "VERSION").upper() == "VERSION":
            os.environ["NCCL_DEBUG"] = "WARN"      # keep stdout to the one JSON line
        dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream(dev)
    ctx = mp.Context(local, stream=stream.cuda_stream)
    ctx.set_timing(True)

    ch = chaingen.make(cfg["chain"])
    assert chaingen.digest(ch) == cfg["digest"], "generator drift"
    a = (cfg["P"], cfg["M"], cfg["beta"], cfg["n_mem"], cfg["n_delay"], cfg["n_periods"])
    dchain = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).to(dev) for k in ("uF", "uB", "W", "a")}
    pinned = {k: torch.from_numpy(np.ascontiguousarray(ch[k])).pin_memory().numpy()
              for k in ("uF", "uB", "W", "a")}
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)

    def step(chain, early_exit=False):
        """One solve; returns (result, this rank's cell updates, launches, step-kernel ms)."""
        if not use_dist:
            if chain is dchain:
                res = ctx.solve_dev(dchain, *a, early_exit=early_exit)
            else:
                res = ctx.solve(chain, *a, early_exit=early_exit)
            cu = res["cell_updates"]
        else:
            res, cu = solve_distributed(chain, *a, early_exit=early_exit, ctx=ctx, device=dev)
        t = ctx.last_timing()
        cnt = ctx.last_counts()
        sb = ctx.last_step_bytes()
        return (res, cu, (cnt["effective_updates"], cnt["useful_updates"], sb["load_bytes"] + sb["store_bytes"]),
                t["launches"], t["step_ms"])

    def timed(chain, k, early_exit=False):
        dev_ms, wall, cus, effs, launches, kern_ms, io = [], [], [], [], 0, 0.0, (0, 0)
        for _ in range(k):
            flush.zero_()
            torch.cuda.synchronize(dev)
            if use_dist:
                dist.barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            w0 = time.perf_counter()
            res, cu, eff, n_l, k_ms = step(chain, early_exit)
            w1 = time.perf_counter()
            e1.record(stream)
            torch.cuda.synchronize(dev)
            dev_ms.append(e0.elapsed_time(e1))
            wall.append(w1 - w0)
            cus.append(cu)
            effs.append(eff)
            launches += n_l
            kern_ms += k_ms
            last_io = ctx.last_io()
            io = (last_io["h2d_bytes"], last_io["d2h_bytes"])
        return dict(res=res, dev_ms=dev_ms, wall=wall, cu=cus, eff=effs, launches=launches,
                    kern_ms=kern_ms, io=io)

    for _ in range(args.warmup):
        step(dchain)
    torch.cuda.synchronize(dev)
    with ClockSampler(local) as clk:
        main_run = timed(dchain, args.steps)
    e2e_run = None if args.no_e2e else timed(pinned, args.steps)
    ee_run = timed(dchain, args.steps, early_exit=True)

    def reduce(x, op):
        if not use_dist:
            return x
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=op)
        return t.item()

    SUM, MAX = (dist.ReduceOp.SUM, dist.ReduceOp.MAX) if use_dist else (None, None)
    K = args.steps
    tot_ms = reduce(sum(main_run["dev_ms"]), MAX)
    cu_step = reduce(main_run["cu"][-1], SUM)
    eff_step = reduce(main_run["eff"][-1][0], SUM)
    useful_step = reduce(main_run["eff"][-1][1], SUM)
    value = cu_step * K / (tot_ms / 1e3)
    kern_ms = reduce(main_run["kern_ms"], MAX)
    launches = int(reduce(main_run["launches"], SUM))
    ttp = reduce(statistics.median(main_run["wall"]), MAX)
    ttp_ee = reduce(statistics.median(ee_run["wall"]), MAX)
    e2e = None
    if e2e_run:
        e2e_ms = reduce(sum(e2e_run["dev_ms"]), MAX)
        e2e_wall = reduce(sum(e2e_run["wall"]), MAX)
        e2e = {"value": cu_step * K / (max(e2e_ms, 1e3 * e2e_wall) / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(reduce(e2e_run["io"][0], SUM)),
               "d2h_bytes_per_step": int(reduce(e2e_run["io"][1], SUM)),
               "ms_per_step": max(e2e_ms, 1e3 * e2e_wall) / K,
               "entry": "madpipe_solve (N=1) / madpipe_sweep+resolve (N>1) on pinned host arrays"}
    if rank != 0:
        if use_dist:
            dist.destroy_process_group()
        return
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    # algorithmic bytes: one fp64 source value per relaxation that must read the table:
    # a live transition (not skipped by delay overflow / C > tau / no fit) whose source row
    # holds a finite value; all-+inf rows and dead transitions read nothing
    # algorithmic bytes of the step kernel: every source-row segment it must
    # bring on chip (one per useful (k, v') of a tile; the two-layer kernel loads a row
    # shared by its two layers once) plus every output row it stores; per GPU
    kbytes_step = reduce(main_run["eff"][-1][2], SUM) / world
    units = useful_step if useful_step > 0 else eff_step
    achieved = kbytes_step * K / (kern_ms / 1e3) / 1e9 if kern_ms > 0 and kbytes_step > 0 else None
    # what a kernel without cross-layer reuse would have to stream for the same relaxations
    streaming = units / world * K * BYTES_PER_UPDATE / (kern_ms / 1e3) / 1e9 if kern_ms > 0 else None
    traffic = None
    prof = os.path.join(ROOT, "profiles", "step_kernel_traffic.json")
    if os.path.exists(prof):
        traffic = json.load(open(prof)).get("dram_bytes_per_launch")
    res = main_run["res"]
    cpu = None
    if world == 1 and not args.no_cpu:
        cpu, _ = oracle_sample(cfg)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": tot_ms / K, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic (chaingen, seeded)",
        "config": {**workload(cfg), "parallelism": ("candidates interleaved over %d rank(s), 1 NCCL "
                                                    "all-reduce(MIN) per solve" % world) if use_dist
                   else "1 GPU, madpipe_solve_dev",
                   "l2": "DP tables >> L2 (%.0f MB per candidate) and a %d MB L2 flush between steps"
                         % ((cfg["L"] + 1) * cfg["P"] * cfg["n_delay"] * cfg["n_mem"] * 8 / 1e6,
                            L2_FLUSH_BYTES >> 20)},
        "time_to_placement_s": ttp, "time_to_placement_early_exit_s": ttp_ee,
        "cell_updates_per_step": cu_step,
        "effective_updates_per_step": eff_step,
        "effective_updates_per_s": eff_step * K / (tot_ms / 1e3),
        "useful_updates_per_step": useful_step,
        "result": {"cand_index": res["cand_index"], "period": res["period"],
                   "special_load": res["special_load"], "n_stages": len(res["stages"])},
        "roofline": {"bound": "hbm", "kernel": ctx.last_kernel(), "achieved": achieved, "peak": hbm_peak,
                     "unit": "GB/s", "frac": (achieved / hbm_peak) if achieved else None,
                     "traffic": traffic, "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured)",
                     "algorithmic_bytes_per_step": kbytes_step,
                     "bytes": "source-row segments loaded + output rows stored by the step kernel",
                     "streaming_equiv": streaming,
                     "streaming_equiv_units": "%d B x %s / step-kernel time" % (
                         BYTES_PER_UPDATE, "useful relaxations" if useful_step > 0 else "effective relaxations"),
                     "kernel_share": kern_ms / tot_ms if tot_ms else None},
        "e2e": e2e, "gpu_launches": launches, "clocks": clk.summary(), "cpu_baseline": cpu,
    }
    print(json.dumps(line), flush=True)
    if use_dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
