#!/usr/bin/env python3
"""Per-CUDA-source-line instruction and stall-sample shares from `ncu -i R --page source --csv --print-source cuda,sass`."""
import csv
import sys
from collections import defaultdict

cur_file = "?"
hdr = None
inst, samp = defaultdict(int), defaultdict(int)
text = {}
line_no = None
for row in csv.reader(open(sys.argv[1])):
    if not row:
        continue
    if row[0] == "File Path":
        cur_file = row[1].split("/")[-1]
        continue
    if row[0] == "Line No":
        hdr = row
        iE = hdr.index("Instructions Executed")
        iS = hdr.index("Warp Stall Sampling (All Samples)")
        continue
    if hdr is None or row[0] == "Function Name":
        continue
    if row[0]:
        line_no = (cur_file, int(row[0]))
        text[line_no] = row[1].strip()[:90]
    try:
        inst[line_no] += int(row[iE] or 0)
        samp[line_no] += int(row[iS] or 0)
    except (ValueError, IndexError):
        pass
ti, ts = sum(inst.values()) or 1, sum(samp.values()) or 1
print(f"total instructions {ti}, stall samples {ts}")
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
for k in sorted(inst, key=lambda k: inst[k] + samp[k] * ti / ts, reverse=True)[:n]:
    print(f"{100 * inst[k] / ti:6.2f}% inst {100 * samp[k] / ts:6.2f}% stall  {k[0]}:{k[1]:<4d} {text.get(k, '')}")
