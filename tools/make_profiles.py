#!/usr/bin/env python
"""Turn the GPU-box captures in gpurun_out/ into committed summaries.

  python tools/make_profiles.py r01 [--bench gpurun_out/bench_bh.json]

writes profiles/<round>/ncu_<workload>_<mode>.md, profiles/<round>/launches_bh.md
and profiles/ncu_counts.json (per workload/mode: DRAM bytes and executed warp
instructions per traversed point, read by bench.py for `traffic` and the
issue-rate roofline).
"""
from __future__ import annotations

import csv
import glob
import io
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import ncu_summary  # noqa: E402

POINTS_RE = re.compile(r'"points_per_rank": (\d+)')


def launches_md(csv_path):
    rows = list(csv.reader(open(csv_path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    agg = {}
    for r in rows[start + 1:]:
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"]
        agg.setdefault(name, []).append(float(d["Metric Value"]))
    tot = sum(sum(v) for v in agg.values())
    out = ["| launches | total us | share | kernel |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        out.append(f"| {len(v)} | {sum(v) / 1e3:.1f} | {100 * sum(v) / tot:.1f}% | `{k[:110]}` |")
    return "\n".join(out)


def main(argv):
    rnd = argv[0]
    outdir = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(outdir, exist_ok=True)
    counts_path = os.path.join(ROOT, "profiles", "ncu_counts.json")
    counts = json.load(open(counts_path)) if os.path.exists(counts_path) else {}
    sys.path.insert(0, ROOT)
    import bench  # noqa: E402
    for rep in sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "prof_*.ncu-rep"))):
        tag = os.path.basename(rep)[len("prof_"):-len(".ncu-rep")]  # e.g. bh_auto
        w, mode = tag.split("_", 1)
        det, raw = ncu_summary.details(rep), ncu_summary.raw(rep)
        lines = [f"# ncu --set full: {tag} (round {rnd})\n",
                 f"source: `{os.path.basename(rep)}` captured by tools/profile_all.sh\n"]
        for k in det:
            d = dict(det[k])
            d.update(raw.get(k, {}))
            lines.append(f"## `{k}`\n")
            lines.append("| metric | value | unit |\n|---|---|---|")
            for m, (v, u) in d.items():
                lines.append(f"| {m} | {v} | {u} |")
            log = os.path.join(ROOT, "gpurun_out", f"ncu_{tag}.log")
            pts = None
            if os.path.exists(log):
                mm = POINTS_RE.search(open(log).read())
                pts = int(mm.group(1)) if mm else None
            def num(key):
                v = d.get(key, (None, ""))[0]
                try:
                    return float(str(v).replace(",", ""))
                except (TypeError, ValueError):
                    return None
            rb, wb = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
            unit_r = d.get("dram__bytes_read.sum", (None, "byte"))[1]
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit_r, 1)
            scale_w = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(
                d.get("dram__bytes_write.sum", (None, "byte"))[1], 1)
            inst = num("smsp__inst_executed.sum")
            dur = num("Duration")
            if pts and rb is not None and inst:
                counts[f"{w}/{mode}"] = {
                    "kernel": k, "points": pts, "round": rnd,
                    "dram_bytes_per_point": (rb * scale + (wb or 0) * scale_w) / pts,
                    "warp_inst_per_point": inst / pts,
                    "ncu_duration": dur, "issue_slots_busy_pct": num("Issue Slots Busy"),
                    "src_sha256": bench.kernel_sha256(w),
                }
        open(os.path.join(outdir, f"ncu_{tag}.md"), "w").write("\n".join(lines) + "\n")
    lb = os.path.join(ROOT, "gpurun_out", "launches_bh.csv")
    if os.path.exists(lb):
        open(os.path.join(outdir, "launches_bh.md"), "w").write(
            f"# Launch list of `python bench.py --steps 2 --warmup 1` under\n"
            f"`ncu --metrics gpu__time_duration.sum --clock-control none` (round {rnd})\n\n"
            "Cold-cache, serialised per-launch times: compare shares, not absolutes.\n\n"
            + launches_md(lb) + "\n")
    json.dump(counts, open(counts_path, "w"), indent=1, sort_keys=True)
    print("wrote", outdir, counts_path)


if __name__ == "__main__":
    main(sys.argv[1:])
