"""Opcode mix of a kernel from its ncu SASS source page (`ncu -i rep --page
source --csv --print-source sass`, gzipped): executed warp instructions and
stall samples per opcode, largest first.
usage: python tools/sass_mix.py profiles/r02/src_bh_auto.csv.gz [top]"""
import csv
import gzip
import io
import sys
from collections import defaultdict

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
rows = list(csv.reader(io.TextIOWrapper(gzip.open(path), encoding="utf-8")))
name = rows[0][1] if rows and rows[0] and rows[0][0] == "Kernel Name" else "?"
hdr = next(r for r in rows if r and r[0] == "Address")
ie, ss = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
agg = defaultdict(lambda: [0, 0])
for r in rows:
    if len(r) < len(hdr) or not r[0].startswith("0x"):
        continue
    src = r[1].strip()
    if src.startswith("@"):
        src = src.split(None, 1)[1] if " " in src else src
    op = src.split()[0].rstrip(";") if src else "?"
    agg[op][0] += int(float(r[ie] or 0))
    agg[op][1] += int(float(r[ss] or 0))
ti = sum(v[0] for v in agg.values()) or 1
ts = sum(v[1] for v in agg.values()) or 1
print(f"# SASS opcode mix: `{name[:90]}`\n")
print(f"source: `{path}`; {ti:.3e} warp instructions, {ts} stall samples\n")
print("| opcode | warp instructions | % | stall samples % |")
print("|---|---|---|---|")
for op, (i, s) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"| `{op}` | {i:.3e} | {100 * i / ti:.1f} | {100 * s / ts:.1f} |")
