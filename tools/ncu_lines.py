"""Aggregate an ncu source page (cuda,sass) per CUDA source line: samples + instructions.
usage: python tools/ncu_lines.py report.ncu-rep [topN]"""
import csv
import subprocess
import sys
from collections import defaultdict

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout.splitlines()
agg = defaultdict(lambda: [0, 0, ""])
fname = ""
hdr = None
for row in csv.reader(out):
    if not row:
        continue
    if row[0] == "File Path":
        fname = row[1].split("/")[-1]
        continue
    if row[0] == "Line No":
        hdr = row
        continue
    if hdr is None:
        continue
    try:
        ln = int(row[0])
    except ValueError:
        continue
    if len(row) < 8 or row[2] != "-":
        continue                       # keep the per-source-line aggregate rows
    try:
        samp = int(row[4] or 0)
        inst = int(row[7] or 0)
    except ValueError:
        continue
    k = (fname, ln)
    agg[k][0] += samp
    agg[k][1] += inst
    agg[k][2] = row[1][:70]
tot_s = sum(v[0] for v in agg.values()) or 1
tot_i = sum(v[1] for v in agg.values()) or 1
print(f"total samples {tot_s} instructions {tot_i}")
for k, v in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{k[0]}:{k[1]:<5} samp {100*v[0]/tot_s:5.1f}%  inst {100*v[1]/tot_i:5.1f}%  {v[2]}")
