#!/usr/bin/env python3
"""N4: the RQ2 trace-size sweep (Fig. 5) on the GPU path.

For the three growth patterns of P:L366 (tracegen configs 6-8: dummy S-box program, thread-distinct
pixels, fixed threads) and input sizes of 10^2..10^6 threads, folds one run on the device and reports the
raw trace (16 B records) against the A-DCFG it becomes (cells, canonical dump bytes): Owl's "merge
duplicate memory accesses" as a compression ratio.  Prints one table (and JSON lines with --json).
"""
import argparse
import json
import os
import struct
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="100,1000,10000,100000,1000000")
    ap.add_argument("--json", action="store_true")
    args = ap.parse_args()
    import torch
    import tracegen
    from paper_conf_dsn_zhaoxcqzj24_b200 import api
    ctx = api.Context(0)
    names = {8: "(1) fixed threads", 6: "(2) S-box lookups", 7: "(3) distinct pixels"}
    print(f"{'pattern':22s} {'threads':>9s} {'records':>11s} {'trace MB':>9s} {'cells':>9s} {'A-DCFG MB':>9s} "
          f"{'ratio':>8s} {'fold ms':>8s}")
    run = 0
    for cfg in (8, 6, 7):
        for t in [int(x) for x in args.sizes.split(",")]:
            p = tracegen.Params.preset(cfg, threads=t)
            segs, n_rec = [], 0
            for m in tracegen.run_segments(p, 0):
                buf, n = tracegen.device_records(p, 0, m.seq)
                segs.append(api.Segment(run, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, n))
                n_rec += n
            torch.cuda.synchronize()
            ctx.ingest(segs)
            ctx.build([run]).destroy()  # warm-up (table sizing)
            ctx.reset_stats()
            g = ctx.build([run])
            st = ctx.stats()
            blob = g.export()
            cells = sum(struct.unpack_from("<4Q", blob, 24))
            row = dict(pattern=names[cfg], config=cfg, threads=t, records=n_rec, trace_bytes=16 * n_rec,
                       cells=cells, adcfg_bytes=len(blob), ratio=16 * n_rec / len(blob), fold_ms=st["last_fold_ms"])
            print(f"{names[cfg]:22s} {t:9d} {n_rec:11d} {16 * n_rec / 1e6:9.2f} {cells:9d} {len(blob) / 1e6:9.3f} "
                  f"{row['ratio']:8.1f} {st['last_fold_ms']:8.3f}")
            if args.json:
                print(json.dumps(row))
            g.destroy()
            ctx.forget_runs([run])
            run += 1


if __name__ == "__main__":
    main()
