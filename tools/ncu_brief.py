"""Key metrics + stall samples + hottest source lines of a one-kernel ncu report:
python tools/ncu_brief.py gpurun_out/full_TAG.ncu-rep [n_lines]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
nl = int(sys.argv[2]) if len(sys.argv) > 2 else 15
raw = list(csv.reader(subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"],
                                     capture_output=True, text=True).stdout.splitlines()))
h, v = raw[0], raw[2]
for w in ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
          "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
          "sm__warps_active.avg.per_cycle_active", "lts__t_sector_hit_rate.pct",
          "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
          "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread"]:
    if w in h:
        print(f"{w:60s} {v[h.index(w)]}")
st = [(int(float(v[i] or 0)), h[i].replace("smsp__pcsamp_warps_issue_stalled_", ""))
      for i in range(len(h)) if h[i].startswith("smsp__pcsamp_warps_issue_stalled_")
      and not h[i].endswith("_not_issued")]
tot = sum(s for s, _ in st) or 1
print("stalls:", ", ".join(f"{n} {100 * s / tot:.0f}%" for s, n in sorted(st, reverse=True)[:9]))
src = list(csv.reader(subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source",
                                      "cuda,sass"], capture_output=True, text=True).stdout.splitlines()))
f, out = "", []
for r in src:
    if r and r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if len(r) > 7 and r[2] == "-":
        try:
            out.append((int(r[4] or 0), int(r[7] or 0), f, int(r[0])))
        except ValueError:
            pass
ts = sum(o[0] for o in out) or 1
ti = sum(o[1] for o in out) or 1
for s, i, f, l in sorted(out, reverse=True)[:nl]:
    print(f"samp {100 * s / ts:5.1f}%  inst {100 * i / ti:5.1f}%  {f}:{l}")
