#!/usr/bin/env python
"""Summarise ncu reports (run here, no GPU): key metrics per kernel -> markdown/JSON.

usage: python tools/ncu_summary.py gpurun_out/prof_bh.ncu-rep [...] [--md out.md] [--json out.json]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "Duration", "SM Frequency", "DRAM Throughput", "Memory Throughput", "L1/TEX Cache Throughput",
    "L2 Cache Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Compute (SM) Throughput", "Issue Slots Busy",
    "Executed Ipc Active", "Warp Cycles Per Issued Instruction", "No Eligible", "Avg. Active Threads Per Warp",
    "Avg. Not Predicated Off Threads Per Warp", "Executed Instructions", "Registers Per Thread",
    "Dynamic Shared Memory Per Block", "Theoretical Occupancy", "Achieved Active Warps Per SM",
    "Block Limit Registers", "Block Limit Shared Mem", "Grid Size", "Block Size",
]
RAW = ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "smsp__inst_executed.sum",
       "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
       "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
       "gpu__time_duration.sum"]


def details(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    res = {}
    for r in csv.DictReader(io.StringIO(out)):
        k = r.get("Kernel Name", "")
        d = res.setdefault(k, {})
        name = r.get("Metric Name")
        if name in KEYS and name not in d:
            d[name] = (r.get("Metric Value"), r.get("Metric Unit"))
    return res


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return {}
    hdr, units = rows[0], rows[1]
    res = {}
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        k = d.get("Kernel Name", "")
        res[k] = {m: (d.get(m), units[hdr.index(m)] if m in hdr else "") for m in RAW if m in d}
    return res


def main(argv):
    reps = [a for a in argv if a.endswith(".ncu-rep")]
    md = argv[argv.index("--md") + 1] if "--md" in argv else None
    js = argv[argv.index("--json") + 1] if "--json" in argv else None
    allres = {}
    lines = []
    for rep in reps:
        det, rw = details(rep), raw(rep)
        for k in det:
            d = dict(det[k])
            d.update({m: v for m, v in rw.get(k, {}).items()})
            allres[f"{rep}::{k}"] = d
            lines.append(f"### `{k}`  ({rep.split('/')[-1]})\n")
            lines.append("| metric | value | unit |\n|---|---|---|")
            for m, (v, u) in d.items():
                lines.append(f"| {m} | {v} | {u} |")
            lines.append("")
    text = "\n".join(lines)
    if md:
        open(md, "w").write(text)
    else:
        print(text)
    if js:
        json.dump(allres, open(js, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1:])
