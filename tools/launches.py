"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list: per
launch (id, kernel, grid, us) and per-kernel totals."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
last = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr, out = None, []
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            v = float(d["Metric Value"].replace(",", ""))
            unit = d.get("Metric Unit", "nsecond")
            us = v / 1000 if unit.startswith("n") else (v * 1000 if unit.startswith("m") else v)
            out.append((d["ID"], d["Kernel Name"][:50], d["Grid Size"], us))
tot = defaultdict(float)
for o in out[-last:]:
    print(f"{o[0]:>5} {o[1]:50s} {o[2]:>14s} {o[3]:10.1f} us")
    tot[o[1]] += o[3]
print("--- totals over the listed launches")
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{k:50s} {v:10.1f} us")
