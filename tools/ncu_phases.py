"""Group an ncu source page by line ranges (phases): python tools/ncu_phases.py rep 'name:a-b,...'"""
import csv
import subprocess
import sys

rep = sys.argv[1]
ranges = []
for tok in sys.argv[2].split(","):
    name, ab = tok.split(":")
    a, b = ab.split("-")
    ranges.append((name, int(a), int(b)))
KF = ["--kernel-name", "regex:" + sys.argv[3]] if len(sys.argv) > 3 else []
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + KF,
                     capture_output=True, text=True).stdout.splitlines()
agg = {n: [0, 0] for n, _, _ in ranges}
agg["other(kernels.cuh)"] = [0, 0]
agg["other files"] = [0, 0]
fname = ""
tot = [0, 0]
for row in csv.reader(out):
    if not row:
        continue
    if row[0] == "File Path":
        fname = row[1]
        continue
    if len(row) < 8 or row[2] != "-":
        continue
    try:
        ln, samp, inst = int(row[0]), int(row[4] or 0), int(row[7] or 0)
    except ValueError:
        continue
    tot[0] += samp
    tot[1] += inst
    key = "other files"
    if fname.endswith("gsnp_kernels.cuh"):
        key = "other(kernels.cuh)"
        for n, a, b in ranges:
            if a <= ln <= b:
                key = n
                break
    agg[key][0] += samp
    agg[key][1] += inst
for k, (s, i) in sorted(agg.items(), key=lambda kv: -kv[1][0]):
    print(f"{k:22s} samples {100 * s / max(tot[0], 1):5.1f}%   instructions {100 * i / max(tot[1], 1):5.1f}%")
