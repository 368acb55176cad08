"""Summarise an ncu --set full report and a launch-list CSV into profiles/.
usage: python tools/ncu_summary.py TAG   (reads gpurun_out/full_TAG.ncu-rep, launches_TAG.csv)"""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]
rep = os.path.join(ROOT, "gpurun_out", f"full_{tag}.ncu-rep")
lcsv = os.path.join(ROOT, "gpurun_out", f"launches_{tag}.csv")
out = []
# ---- launch list (ncu --metrics gpu__time_duration.sum)
agg = defaultdict(lambda: [0, 0.0])
hdr = None
for r in csv.reader(open(lcsv)):
    if r and r[0] == "ID":
        hdr = r
        continue
    if not hdr or len(r) < len(hdr):
        continue
    d = dict(zip(hdr, r))
    if d.get("Metric Name") != "gpu__time_duration.sum":
        continue
    k = d["Kernel Name"].split("(")[0]
    agg[k][0] += 1
    agg[k][1] += float(d["Metric Value"])
tot = sum(v[1] for v in agg.values())
out.append(f"# ncu summary — {tag}\n")
out.append("## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, "
           "`python bench.py --steps 2 --warmup 1 --no-cpu`; cold-cache, serialised — compare shares)\n")
out.append("| kernel | launches | total ms | share |\n|---|---|---|---|")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
    out.append(f"| {k} | {v[0]} | {v[1] / 1e6:.3f} | {100 * v[1] / tot:.1f}% |")
# ---- full capture
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                     text=True).stdout.splitlines()
rows = list(csv.reader(raw))
h = rows[0]
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.per_cycle_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum"]
units = rows[1]
traffic = {}
for v in rows[2:]:
    d = dict(zip(h, v))
    u = dict(zip(h, units))
    name = d["Kernel Name"].split("(")[0]
    out.append(f"\n## `{name}` (`ncu --set full`, C2 48 Mb 20X, tools/profile_call.py)\n")
    out.append("| metric | value |\n|---|---|")
    for k in keys:
        if k in d:
            out.append(f"| {k} | {d[k]} {u.get(k, '')} |")
    st = sorted([(float(d[k]), k) for k in d if k.startswith("smsp__pcsamp_warps_issue_stalled")
                 and not k.endswith("not_issued") and d[k] not in ("", "0")], reverse=True)[:8]
    tot_s = sum(x for x, _ in st) or 1
    out.append("\nTop stall reasons (PC samples): " + ", ".join(
        f"{k.replace('smsp__pcsamp_warps_issue_stalled_', '')} {100 * x / tot_s:.0f}%" for x, k in st))

    def tobytes(val, unit):
        f = float(val)
        return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
    if "k_call_tile" in name and "dram__bytes_read.sum" in d:
        traffic = {"workload": "C2", "kernel": name,
                   "bytes_per_launch": tobytes(d["dram__bytes_read.sum"], u["dram__bytes_read.sum"]) +
                   tobytes(d["dram__bytes_write.sum"], u["dram__bytes_write.sum"]),
                   "source": f"profiles/ncu_{tag}.md (ncu --set full)"}
open(os.path.join(ROOT, "profiles", f"ncu_{tag}.md"), "w").write("\n".join(out) + "\n")
if traffic:
    json.dump(traffic, open(os.path.join(ROOT, "profiles", "call_tile_dram_bytes.json"), "w"), indent=1)
print("\n".join(out))
