#!/usr/bin/env python
"""Summarise ncu captures brought back in gpurun_out/ into profiles/ (tracked).

  python scripts/summarize_ncu.py --rep gpurun_out/prof_lane.ncu-rep --tag r01_lane
  python scripts/summarize_ncu.py --launches gpurun_out/launches.csv --tag r01

For a --set full report it writes profiles/<tag>_ncu_full.json (per kernel:
duration, DRAM bytes, issue/warp efficiency, occupancy, top stall reasons,
instructions per event) and, with --traffic, profiles/ncu_full_summary.json
(the per-launch DRAM traffic bench.py reports as roofline.traffic).  For a
launch list it writes profiles/<tag>_launches.json (per kernel name: count,
total and mean device time, share of the listed time).
"""
import argparse
import csv
import re
import io
import json
import os
import statistics
import subprocess
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.environ.get("NCU_SUMMARY_DIR") or os.path.join(ROOT, "profiles")
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "smsp__thread_inst_executed_per_inst_executed.ratio",
        "smsp__warps_eligible.avg.per_cycle_active", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "launch__occupancy_limit_shared_mem",
        "launch__occupancy_limit_registers", "launch__grid_size", "launch__block_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sectors.sum",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed"]
TO_BYTES = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def full(rep, tag, events_per_launch, traffic, workload, traces, only=None):
    hdr, units, data = raw(rep)
    idx = {h: i for i, h in enumerate(hdr)}
    kernels = []
    for r in data:
        if only and not re.search(only, r[idx["Kernel Name"]]):
            continue
        k = {"kernel": r[idx["Kernel Name"]]}
        for key in KEYS:
            if key in idx:
                k[key] = {"value": r[idx[key]], "unit": units[idx[key]]}
        rd = float(r[idx["dram__bytes_read.sum"]]) * TO_BYTES[units[idx["dram__bytes_read.sum"]]]
        wr = float(r[idx["dram__bytes_write.sum"]]) * TO_BYTES[units[idx["dram__bytes_write.sum"]]]
        k["dram_bytes_per_launch"] = rd + wr
        if "smsp__inst_executed.sum" in idx and events_per_launch:
            k["warp_instructions_per_event"] = float(r[idx["smsp__inst_executed.sum"]]) / events_per_launch
        stalls = {h[len("smsp__pcsamp_warps_issue_stalled_"):]: float(r[idx[h]] or 0)
                  for h in hdr if h.startswith("smsp__pcsamp_warps_issue_stalled_")
                  and not h.endswith("_not_issued")}
        tot = sum(stalls.values()) or 1.0
        k["stall_share_top"] = {s: round(v / tot, 3) for s, v in
                                sorted(stalls.items(), key=lambda x: -x[1])[:6]}
        kernels.append(k)
    doc = {"report": os.path.basename(rep), "capture": "ncu --set full --clock-control none "
           "--import-source on, one launch per policy of bench.py --profile (c2 10^6 x 64)",
           "events_per_launch": events_per_launch, "kernels": kernels}
    with open(os.path.join(PROF, f"{tag}_ncu_full.json"), "w") as f:
        json.dump(doc, f, indent=1)
    if traffic:
        per = [k["dram_bytes_per_launch"] for k in kernels]
        with open(os.path.join(PROF, "ncu_full_summary.json"), "w") as f:
            json.dump({"workload": workload, "traces": traces, "source": f"{tag}_ncu_full.json",
                       "dram_bytes_per_launch": statistics.mean(per),
                       "per_kernel": {k["kernel"]: k["dram_bytes_per_launch"] for k in kernels},
                       "limiter": {k["kernel"]: {
                           "warp_instructions_per_event": round(k.get("warp_instructions_per_event", 0), 2),
                           "issue_active_pct": float(k["smsp__issue_active.avg.pct_of_peak_sustained_active"]["value"]),
                           "active_lanes": float(k["smsp__thread_inst_executed_per_inst_executed.ratio"]["value"]),
                           "alu_pipe_pct": float(k["sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"]["value"]),
                           "top_stalls": k["stall_share_top"]} for k in kernels}},
                      f, indent=1)


def launches(path, tag):
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    rows = list(csv.reader(lines))
    hdr = rows[0]
    ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = defaultdict(list)
    for r in rows[1:]:
        v = float(r[iv].replace(",", ""))
        v = v / 1e3 if r[iu] == "ns" else (v if r[iu] == "us" else v * 1e3)
        agg[r[ik]].append(v)
    total = sum(sum(v) for v in agg.values())
    doc = {"source": os.path.basename(path), "note": "cold-cache serialised ncu times; compare shares",
           "total_us": total,
           "kernels": {k: {"count": len(v), "total_us": sum(v), "mean_us": statistics.mean(v),
                           "share": sum(v) / total} for k, v in
                       sorted(agg.items(), key=lambda x: -sum(x[1]))}}
    with open(os.path.join(PROF, f"{tag}_launches.json"), "w") as f:
        json.dump(doc, f, indent=1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rep")
    ap.add_argument("--launches")
    ap.add_argument("--tag", required=True)
    ap.add_argument("--events", type=float, default=3.2e8)
    ap.add_argument("--traffic", action="store_true")
    ap.add_argument("--workload", default="c2_1e6x64_rho2")
    ap.add_argument("--traces", type=int, default=1_000_000)
    ap.add_argument("--only", default=None, help="regex: summarise only these kernels (e.g. the "
                    "compact kernel's first pass, not its 17-bit / 32-bit fallback passes)")
    a = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    if a.rep:
        full(a.rep, a.tag, a.events, a.traffic, a.workload, a.traces, a.only)
    if a.launches:
        launches(a.launches, a.tag)


if __name__ == "__main__":
    main()
