#!/usr/bin/env python3
"""Hottest SASS instructions (by instructions executed) of an `ncu --page source --csv --print-source cuda,sass`
export, in address order, with their source line and stall samples: the per-chunk instruction budget at a glance.
usage: ncu_sass_hot.py src.csv [min_share_of_max]"""
import csv
import sys

rows, line = [], None
hdr = None
for row in csv.reader(open(sys.argv[1])):
    if not row:
        continue
    if row[0] == "Line No":
        hdr = row
        continue
    if hdr is None or row[0] in ("File Path", "Function Name"):
        continue
    if row[0]:
        line = row[0]
        continue
    if row[2].startswith("0x"):
        try:
            ex = int(row[hdr.index("Instructions Executed")] or 0)
            st = int(row[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
        except ValueError:
            continue
        rows.append((int(row[2], 16), line, row[3].strip(), ex, st))
mx = max(r[3] for r in rows)
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
tot = sum(r[3] for r in rows)
sel = [r for r in sorted(rows) if r[3] >= thr * mx]
print(f"total executed {tot}, max {mx}, {len(sel)} instructions >= {thr} x max, their share {sum(r[3] for r in sel) / tot:.3f}")
for a, ln, t, ex, st in sel:
    print(f"{a & 0xFFFFF:6x} L{ln:>4} {ex / mx:5.2f} st {st:6d}  {t[:90]}")
