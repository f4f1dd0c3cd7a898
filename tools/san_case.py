#!/usr/bin/env python3
"""One small build + diff + leak test through the C ABI, for compute-sanitizer runs (tools/gpu_san.sh):
C1 at full size and a C2 slice (grid_div 64), warp-major and channel order (folded in place through the burst index,
and copied to warp-major order), plus config 9 (kernel sequences)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import tracegen  # noqa: E402
from paper_conf_dsn_zhaoxcqzj24_b200 import api  # noqa: E402

# last field: 0 warp-major, 1 channel order in place (the default), 2 channel order copied
CASES = ((1, 1, 10, 10, 0), (2, 64, 2, 2, 0), (2, 64, 1, 1, 1), (2, 64, 1, 1, 2), (9, 16, 2, 3, 0))
if os.environ.get("SAN_CASES"):  # e.g. "3:8:2:2,5:16:2:2" = config:grid_div:runs_fix:runs_rnd (warp-major)
    CASES = tuple(tuple(int(x) for x in c.split(":")) + (0,) for c in os.environ["SAN_CASES"].split(","))

ctx = api.Context(0)
for cfg, div, nf, nr, inter in CASES:
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=nf, runs_rnd=nr)
    ctx.set_config(channel_order=api.OWL_CHANNEL_COPY if inter == 2 else 0)
    segs = []
    for r in range(p.n_runs):
        for m in tracegen.run_segments(p, r):
            if inter:
                rec = tracegen.interleave(tracegen.host_records(p, r, m.seq))
                buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
                segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, len(rec), flags=0))
            else:
                buf, n = tracegen.device_records(p, r, m.seq)
                segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, n))
    ctx.ingest(segs)
    runs = list(range(p.n_runs))
    ef = ctx.build([r for r in runs if tracegen.run_class(p, r) == 0])
    er = ctx.build([r for r in runs if tracegen.run_class(p, r) == 1])
    d, lk = ctx.diff(ef, er), ctx.leak_test(ef, er, 0.05)
    mode = ("warp-major", "channel in place", "channel copy")[inter]
    print(f"C{cfg} div {div} {mode}: {len(d)} diff rows, {len(lk)} leaks", flush=True)
    ef.destroy(); er.destroy()
    ctx.forget_runs(runs)
