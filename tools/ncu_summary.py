#!/usr/bin/env python3
"""One-screen summary of an `ncu --set full` report (the metrics SURVEY §8(d) asks for), per profiled launch.

usage: ncu -i prof.ncu-rep --page raw --csv > raw.csv; python tools/ncu_summary.py raw.csv [records_per_launch]
"""
import csv
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum", "lts__t_sector_hit_rate.pct",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "smsp__inst_executed.sum", "smsp__thread_inst_executed.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic", "sm__cycles_elapsed.avg.per_second",
]
lines = [l for l in open(sys.argv[1]) if not l.startswith("==")]
rows = list(csv.reader(lines))
h, units = rows[0], rows[1]
nrec = float(sys.argv[2]) if len(sys.argv) > 2 else None
for v in rows[2:]:
    name = v[h.index("Kernel Name")] if "Kernel Name" in h else "?"
    print(f"== {name[:100]}")
    vals = {}
    for k in KEYS:
        if k in h:
            i = h.index(k)
            print(f"  {k:62s} {v[i]:>18s} {units[i]}")
            try:
                vals[k] = float(v[i].replace(",", ""))
            except ValueError:
                pass
    stalls = []
    for i, k in enumerate(h):
        if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
            try:
                stalls.append((float(v[i].replace(",", "")), k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            except ValueError:
                pass
    stalls.sort(reverse=True)
    print("  stalls per issue: " + ", ".join(f"{n} {x:.2f}" for x, n in stalls[:8]))
    if nrec:
        t = vals.get("gpu__time_duration.sum")
        unit = units[h.index("gpu__time_duration.sum")]
        t_s = t * (1e-3 if unit == "ms" else 1e-6 if unit == "us" else 1e-9 if unit == "ns" else 1.0)
        rd = vals.get("dram__bytes_read.sum", 0)
        ru = units[h.index("dram__bytes_read.sum")]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(ru, 1)
        print(f"  records {nrec:.4g}: {nrec / t_s:.4g} records/s, algorithmic {16 * nrec / t_s / 1e9:.1f} GB/s, "
              f"dram read {rd * scale / (16 * nrec):.3f} x algorithmic, "
              f"{vals.get('smsp__inst_executed.sum', 0) / nrec:.2f} warp-inst/record")
