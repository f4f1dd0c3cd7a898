#!/usr/bin/env python3
"""N2 measurement: the same C2 runs ingested warp-major vs channel-order (bursts of 32 records, warps
round-robin: what a tracer's channel delivers, reading R17).  Prints build time and records/s of each."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch

    import tracegen
    from paper_conf_dsn_zhaoxcqzj24_b200 import api
    p = tracegen.Params.preset(2, runs_fix=2, runs_rnd=2)
    runs = [0, 2]  # two FIX runs (one class)
    ctx = api.Context(0)
    segs, n_rec, keep = [], 0, []
    for r in runs:
        for m in tracegen.run_segments(p, r):
            host = tracegen.host_records(p, r, m.seq)
            for k, rec in ((0, host), (1, tracegen.interleave(host))):
                buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
                keep.append(buf)
                flags = api.OWL_SEG_WARP_MAJOR if k == 0 else 0
                segs.append(api.Segment(r + 1000 * k, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, len(rec),
                                        flags=flags))
            n_rec += len(host)
    ctx.ingest(segs)
    for name, rs in (("warp-major", runs), ("channel-order", [r + 1000 for r in runs])):
        ctx.build(rs).destroy()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(3):
            ctx.build(rs).destroy()
        torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / 3
        print(f"{name:14s} {n_rec} records  build {dt * 1e3:8.2f} ms  {n_rec / dt:.3g} records/s")


if __name__ == "__main__":
    main()
