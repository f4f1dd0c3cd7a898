#!/usr/bin/env python3
"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: per-kernel launches, total time, share."""
import csv
import sys
from collections import defaultdict

lines = [l for l in open(sys.argv[1]) if not l.startswith("==")]
rows = list(csv.DictReader(lines))
skip = sys.argv[2].split(",") if len(sys.argv) > 2 else ["og_"]  # generator kernels (untimed setup)
t, c = defaultdict(float), defaultdict(int)
for r in rows:
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    name = r["Kernel Name"].split("(")[0]
    if any(name.startswith(s) for s in skip):
        continue
    t[name] += float(r["Metric Value"].replace(",", "")) * (1e-3 if r["Metric Unit"] == "ns" else 1.0)
    c[name] += 1
tot = sum(t.values())
print(f"{'kernel':70s} {'launches':>8s} {'total_us':>12s} {'share':>7s}")
for k in sorted(t, key=t.get, reverse=True):
    print(f"{k[:70]:70s} {c[k]:8d} {t[k]:12.1f} {100 * t[k] / tot:6.2f}%")
print(f"{'TOTAL (excluding generator kernels)':70s} {sum(c.values()):8d} {tot:12.1f}")
