"""Top SASS regions for one stall reason: python tools/ncu_stall.py rep stall_no_inst [N]"""
import csv
import subprocess
import sys

rep, col = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
KF = ["--kernel-name", "regex:" + sys.argv[4]] if len(sys.argv) > 4 else []
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + KF,
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out))
hdr = None
fname = ""
res = []
cur_src = ""
for row in rows:
    if not row:
        continue
    if row[0] == "File Path":
        fname = row[1].split("/")[-1]
        continue
    if row[0] == "Line No":
        hdr = row
        ci = hdr.index(col)
        continue
    if hdr is None or len(row) <= ci:
        continue
    if row[2] == "-":
        cur_src = f"{fname}:{row[0]} {row[1][:50]}"
        continue
    try:
        v = float(row[ci] or 0)
    except ValueError:
        continue
    res.append((v, row[2][-6:], row[3][:50], cur_src))
tot = sum(r[0] for r in res) or 1
print(f"total {col}: {tot}")
for v, a, s, src in sorted(res, reverse=True)[:top]:
    print(f"{100*v/tot:5.1f}% {a} {s:50s} | {src}")
