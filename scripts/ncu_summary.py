"""Summarise ncu outputs into profiles/ (tracked evidence for the bench's roofline).

    python scripts/ncu_summary.py launches <launches.csv> <out.md>
        per-kernel share of the device time from an `ncu --metrics gpu__time_duration.sum` launch list
    python scripts/ncu_summary.py full <prof.ncu-rep> <out.md> [--pipes-json profiles/r02b_step_pipes.json]
        key metrics + top stall reasons + hottest SASS lines of a `--set full` capture; the
        pipe utilisations of the (first) captured launch go to the JSON the bench reads
    python scripts/ncu_summary.py traffic <dram.csv> <one_solve.json> <out.json>
        DRAM bytes of EVERY step-kernel launch of one GPT sweep (ncu --metrics
        dram__bytes_read.sum,dram__bytes_write.sum -k regex:pair_step on scripts/gpt_one_sweep.py)
        against that sweep's algorithmic byte counts
"""
from __future__ import annotations

import collections
import csv
import io
import json
import subprocess
import sys

NCU = "/usr/local/cuda/bin/ncu"

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__t_sector_hit_rate.pct",
    "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem",
    "launch__occupancy_limit_registers", "sm__cycles_elapsed.avg",
]


def _to_ns(v, unit):
    v = float(v.replace(",", ""))
    return v * {"ns": 1, "nsecond": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(unit, 1)


def launches(csv_path, out_md):
    rows = list(csv.reader(open(csv_path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    tot, cnt = collections.Counter(), collections.Counter()
    for r in rows[hi + 1:]:
        if len(r) <= vi or not r[vi]:
            continue
        name = r[ki].split("(")[0].replace("void ", "")
        tot[name] += _to_ns(r[vi], r[ui])
        cnt[name] += 1
    T = sum(tot.values())
    lines = ["# ncu launch list: per-kernel device time (cold-cache, serialised)", "",
             "source: `%s`" % csv_path, "", "| kernel | launches | total ms | share |", "|---|---|---|---|"]
    for k, v in tot.most_common():
        lines.append("| %s | %d | %.3f | %.4f |" % (k, cnt[k], v / 1e6, v / T))
    lines.append("")
    lines.append("total %.3f ms over %d launches" % (T / 1e6, sum(cnt.values())))
    open(out_md, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


PIPES = {"fp64_pct": "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
         "alu_pct": "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
         "lsu_pct": "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
         "issue_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
         "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
         "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"}


def traffic(csv_path, solve_json, out_json):
    rows = list(csv.reader(open(csv_path)))
    hi = next(i for i, r in enumerate(rows) if "Metric Name" in r)
    h = rows[hi]
    ni, vi, ui, ki = h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit"), h.index("Kernel Name")
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    tot, ns, ids = 0.0, 0.0, set()
    for r in rows[hi + 1:]:
        if len(r) <= vi or "pair_step" not in r[ki]:
            continue
        if r[ni].startswith("dram__bytes"):
            tot += float(r[vi].replace(",", "")) * scale[r[ui]]
            ids.add(r[0])
        elif r[ni] == "gpu__time_duration.sum":
            ns += _to_ns(r[vi], r[ui])
    s = json.load(open(solve_json))
    out = {"dram_bytes_per_solve": tot, "step_launches_per_solve": len(ids), "step_ns_cold_serialised": ns,
           "moved_bytes_per_solve": s["moved_bytes"], "compulsory_bytes_per_solve": s["compulsory_bytes"],
           "traffic_over_moved": tot / s["moved_bytes"], "traffic_over_compulsory": tot / s["compulsory_bytes"],
           "source": csv_path, "note": "sum over every pair_step_kernel launch of one full GPT sweep "
                                       "(scripts/gpt_one_sweep.py under ncu; cold-cache, serialised)"}
    json.dump(out, open(out_json, "w"), indent=1)
    print(json.dumps(out, indent=1))


def full(rep, out_md, pipes_json=None):
    raw = subprocess.run([NCU, "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, units = rows[0], rows[1]
    idx = {n: i for i, n in enumerate(h)}
    lines = ["# ncu --set full summary", "", "source: `%s`" % rep, ""]
    traffic = []
    pipes = None
    for r in rows[2:]:
        name = r[idx["Kernel Name"]] if "Kernel Name" in idx else "?"
        lines += ["## %s" % name[:120], "", "| metric | value | unit |", "|---|---|---|"]
        for k in KEYS:
            if k in idx:
                lines.append("| %s | %s | %s |" % (k, r[idx[k]], units[idx[k]]))
        if pipes is None:
            pipes = {key: float(r[idx[m]].replace(",", "")) for key, m in PIPES.items() if m in idx}
            pipes["kernel"] = name[:80]
        st = sorted(((float(r[i].replace(",", "") or 0), n) for n, i in idx.items()
                     if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio")),
                    reverse=True)[:8]
        lines += ["", "top stall reasons (warps stalled per issue):", ""]
        lines += ["- %s: %.3f" % (n.replace("smsp__average_warps_issue_stalled_", "").replace(
            "_per_issue_active.ratio", ""), v) for v, n in st]
        lines.append("")
        try:
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            rd = float(r[idx["dram__bytes_read.sum"]].replace(",", "")) * scale[units[idx["dram__bytes_read.sum"]]]
            wr = float(r[idx["dram__bytes_write.sum"]].replace(",", "")) * scale[units[idx["dram__bytes_write.sum"]]]
            traffic.append(rd + wr)
        except (KeyError, ValueError):
            pass
    sass = subprocess.run([NCU, "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                          capture_output=True, text=True).stdout
    srows = list(csv.reader(io.StringIO(sass)))
    try:
        hi = next(i for i, r in enumerate(srows) if r and r[0] == "Address")
        sh = srows[hi]
        iS, iW = sh.index("Source"), sh.index("Warp Stall Sampling (All Samples)")
        data = [r for r in srows[hi + 1:] if len(r) > iW]
        tot = sum(float(r[iW] or 0) for r in data) or 1.0
        lines += ["hottest SASS (share of warp-stall samples):", "", "```"]
        for r in sorted(data, key=lambda r: -float(r[iW] or 0))[:15]:
            lines.append("%6.2f%%  %s" % (100 * float(r[iW]) / tot, r[iS][:100]))
        lines.append("```")
    except StopIteration:
        pass
    open(out_md, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines[:60]))
    if pipes_json and pipes:
        pipes["source"] = rep
        pipes["dram_bytes_captured_launch"] = traffic[0] if traffic else None
        json.dump(pipes, open(pipes_json, "w"), indent=1)


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3])
    elif sys.argv[1] == "traffic":
        traffic(sys.argv[2], sys.argv[3], sys.argv[4])
    else:
        pj = sys.argv[sys.argv.index("--pipes-json") + 1] if "--pipes-json" in sys.argv else None
        full(sys.argv[2], sys.argv[3], pj)
