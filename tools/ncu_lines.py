"""Aggregate an ncu report's per-instruction counters by CUDA source line.
usage: python tools/ncu_lines.py report.ncu-rep [top_n]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fname = "?"
agg = {}
hdr = None
for r in csv.reader(io.StringIO(out)):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < len(hdr) or not r[0].isdigit():
        continue
    def num(x):
        try:
            return float(x)
        except ValueError:
            return 0.0
    st = num(r[4])
    ex = num(r[7])
    key = (fname, int(r[0]))
    a = agg.setdefault(key, [0.0, 0.0, r[1]])
    a[0] += st
    a[1] += ex
tot_st = sum(v[0] for v in agg.values()) or 1
tot_ex = sum(v[1] for v in agg.values()) or 1
print(f"total stall samples {tot_st:.0f}, instructions {tot_ex:.3e}")
for (f, ln), (st, ex, src) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top]:
    print(f"{100*ex/tot_ex:5.1f}% inst {100*st/tot_st:5.1f}% stall {f}:{ln:<4} {src.strip()[:90]}")
