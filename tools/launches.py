"""Print an ncu launch-list CSV (gpu__time_duration.sum) one launch per line: python tools/launches.py f.csv"""
import csv
import sys

hdr = None
for r in csv.reader(open(sys.argv[1])):
    if r and r[0] == "ID":
        hdr = r
        continue
    if not hdr or len(r) < len(hdr):
        continue
    d = dict(zip(hdr, r))
    if d.get("Metric Name") == "gpu__time_duration.sum":
        print(f'{d["ID"]:>4} {d["Kernel Name"].split("(")[0]:28s} grid {d.get("Grid Size", ""):>16s} '
              f'{float(d["Metric Value"]):10.1f} {d.get("Metric Unit", "")}')
