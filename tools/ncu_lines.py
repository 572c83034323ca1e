"""Warp-stall samples and executed instructions per CUDA source line from an ncu report.
usage: python tools/ncu_lines.py REPORT.ncu-rep [n_top]"""
import csv
import io
import os
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
isamp = iex = None
fname = "?"
agg = []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = os.path.basename(r[1])
        continue
    if r[0] == "Line No":
        isamp = r.index("Warp Stall Sampling (All Samples)")
        iex = r.index("Instructions Executed")
        continue
    if isamp is None or not r[0].strip().isdigit():
        continue
    try:
        agg.append((float(r[isamp] or 0), float(r[iex] or 0), fname, int(r[0]), r[1].strip()[:88]))
    except ValueError:
        pass
tot = sum(a[0] for a in agg) or 1
for s, e, f, ln, src in sorted(agg, key=lambda a: -a[0])[:ntop]:
    print(f"{f[:14]:14s} L{ln:4d} {s/tot*100:5.1f}% {e/1e6:7.2f}M  {src}")
