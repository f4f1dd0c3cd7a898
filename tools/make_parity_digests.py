#!/usr/bin/env python3
"""Full-size parity fixtures, computed by the CPU ORACLE ONLY (oracle/ + the seeded generator tracegen/):

    python tools/make_parity_digests.py [--configs 1,2,3,4,5] [--batch 16]

For each BASELINE.json config at its full size (tracegen presets: C1 20 runs ... C5 1000 runs) the runs are
generated on the host in batches of ascending run ids and merged into E_fix / E_rnd with the oracle's
incremental evidence (O1-O4, oracle.Evidence: the same result as one build over all runs, checked by
tests/test_oracle_incremental.py), so no more than one batch of records is ever in host memory.  Written:

  tests/golden/full_size/C<k>.json   SHA-256 of the canonical dumps of E_fix and E_rnd and of the diff rows
                                    (A5), record / cell / row counts, the oracle's wall time and thread count
  tests/golden/full_size/C<k>.npz    every KS row (O7, exact fields + D bits, p, fail) and every leak row (O6/O8)

tests/test_gpu_full_size.py builds the same configurations on the GPU (through the C ABI, in the bench's
launch configuration) and compares.  No value here comes from the CUDA path.
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import tracegen  # noqa: E402
from oracle import oracle  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "full_size")


def digest_config(cfg: int, batch: int, threads: int) -> None:
    p = tracegen.Params.preset(cfg)
    t0 = time.perf_counter()
    ev = {0: oracle.Evidence(0), 1: oracle.Evidence(1)}
    n_rec = 0
    runs = list(range(p.n_runs))
    for k in range(0, len(runs), batch):
        by_cls = {0: [], 1: []}
        for r in runs[k:k + batch]:
            for m in tracegen.run_segments(p, r):
                rec = tracegen.host_records(p, r, m.seq, threads)
                n_rec += len(rec)
                by_cls[m.input_class].append(oracle.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, rec))
        for c in (0, 1):
            if by_cls[c]:
                ev[c].add(by_cls[c], threads)
        del by_cls
        print(f"C{cfg}: {min(k + batch, len(runs))}/{len(runs)} runs, {n_rec} records, "
              f"{time.perf_counter() - t0:.0f} s", flush=True)
    f, r = ev[0], ev[1]
    bf, br = f.export(), r.export()
    diff = oracle.diff(f, r)
    ks = oracle.ks_tests(f, r, 0.05)
    leaks = oracle.leak_test(f, r, 0.05)
    dt = time.perf_counter() - t0
    doc = {
        "_source": "tools/make_parity_digests.py: CPU oracle (oracle/owl_oracle.cpp) on the seeded generator "
                   "(tracegen/), incremental evidence; no value from the CUDA path",
        "config": cfg, "workload": tracegen.CONFIG_NAMES[cfg], "runs_fix": p.runs_fix, "runs_rnd": p.runs_rnd,
        "records": n_rec, "oracle_seconds": round(dt, 1), "oracle_threads": threads,
        "e_fix_sha256": hashlib.sha256(bf).hexdigest(), "e_fix_bytes": len(bf),
        "e_rnd_sha256": hashlib.sha256(br).hexdigest(), "e_rnd_bytes": len(br),
        "diff_rows": int(len(diff)), "diff_sha256": hashlib.sha256(diff.tobytes()).hexdigest(),
        "ks_rows": int(len(ks)), "leak_rows": int(len(leaks)),
    }
    os.makedirs(OUT, exist_ok=True)
    with open(os.path.join(OUT, f"C{cfg}.json"), "w") as fh:
        json.dump(doc, fh, indent=1)
        fh.write("\n")
    np.savez_compressed(os.path.join(OUT, f"C{cfg}.npz"), ks=ks, leaks=leaks)
    print(json.dumps(doc), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="1,2,3,4,5")
    ap.add_argument("--batch", type=int, default=16, help="runs per batch (host memory bound)")
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 1)
    a = ap.parse_args()
    for cfg in (int(c) for c in a.configs.split(",")):
        digest_config(cfg, a.batch, a.threads)


if __name__ == "__main__":
    main()
