#!/usr/bin/env python3
"""Benchmark of the Owl hot path on B200: trace records/s into A-DCFG + leak tests (BASELINE.json metric).

A step = one pass of the whole hot path over the workload: fold + Myers-merge every
run of both input classes into E_fix and E_rnd (owl_build_adcfg), diff them (owl_diff_adcfg) and run the
kernel / KS leak tests with localization (owl_leak_test).  Records are generated on the device (untimed)
and stay resident in HBM; the workload (44.5 GB at N=1) is far larger than the 126 MB L2, so no flush is
needed between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2] [--impl ours|reference]

Prints ONE JSON line (rank 0).  Multi-GPU: one process per GPU (torchrun), runs sharded across ranks
(weak scaling: every rank holds the same number of runs of both classes), one key-hash exchange of the
partial evidences (NCCL all_to_all_single), owner-side KS tests, leak rows gathered to rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "trace records/sec into A-DCFG + leak tests at 1/2/4/8 B200; % HBM peak"


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            pk = json.load(f)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    except Exception:  # noqa: BLE001
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def _traffic(records_per_launch):
    """DRAM bytes (read + write) per fold launch from the committed ncu --set full capture
    (profiles/fold_traffic.json, written from the capture named there), scaled to this launch's records."""
    try:
        with open(os.path.join(ROOT, "profiles", "fold_traffic.json")) as f:
            t = json.load(f)
        return t["traffic_bytes_per_launch"] / t["records_per_launch"] * records_per_launch
    except Exception:  # noqa: BLE001
        return None


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index, self.rows, self.proc = index, [], None
        self.window, self._seen = False, False

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:  # noqa: BLE001
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self._seen = True
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 7 and self.window:
                self.rows.append(parts)

    def wait_ready(self, timeout=10.0):
        """nvidia-smi needs ~0.5-1 s to start: wait until it prints, so the timed region is covered."""
        t0 = time.time()
        while self.proc and not self._seen and time.time() - t0 < timeout and self.proc.poll() is None:
            time.sleep(0.05)

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:  # noqa: BLE001
            self.proc.kill()
        sm = sorted(float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit())
        mx = max((float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()), default=None)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(self.rows)}


def _dist():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def _class_runs(p, runs, cls):
    import tracegen
    return [r for r in runs if tracegen.run_class(p, r) == cls]


def cpu_baseline(cfg: int, target_s: float = 15.0):
    """The oracle as it stands on the host cores, on a bounded sample of the same workload."""
    import tracegen
    from oracle import oracle
    threads = os.cpu_count() or 1
    div = {1: 1, 2: 16, 3: 8, 4: 64, 5: 16}[cfg]
    runs = 2
    while True:
        p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=runs, runs_rnd=runs)
        segs, _ = oracle.run_config(p, threads=threads)
        n = sum(len(s.records) for c in (0, 1) for s in segs[c])
        t0 = time.perf_counter()
        f, r = oracle.build(segs[0], threads), oracle.build(segs[1], threads)
        oracle.diff(f, r)
        oracle.leak_test(f, r, 0.05)
        dt = time.perf_counter() - t0
        if dt >= target_s / 4 or runs >= 64:
            break
        runs = min(64, max(runs * 2, int(runs * target_s / max(dt, 1e-3) / 2)))
    return {"value": n / dt, "unit": "records/s", "cores": threads, "kind": "oracle",
            "sample": f"config C{cfg} grid_div={div} runs={2 * runs} ({n} records, {dt:.1f} s, build E_fix+E_rnd+diff+leak test)"}


def run_reference(args):
    world, rank, _ = _dist()
    if rank != 0:
        return
    import tracegen
    from oracle import oracle
    threads = os.cpu_count() or 1
    cfg = args.config
    div = {1: 1, 2: 32, 3: 16, 4: 128, 5: 32}[cfg]
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=2, runs_rnd=2)
    segs, _ = oracle.run_config(p, threads=threads)
    n = sum(len(s.records) for c in (0, 1) for s in segs[c])

    def step():
        f, r = oracle.build(segs[0], threads), oracle.build(segs[1], threads)
        oracle.diff(f, r)
        oracle.leak_test(f, r, 0.05)

    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = (time.perf_counter() - t0) / args.steps
    v = n / dt
    sample = f"config C{cfg} grid_div={div}, 2+2 runs ({n} records) per step"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": v, "unit": "records/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": tracegen.CONFIG_NAMES[cfg], "sample": sample},
        "cpu_baseline": {"value": v, "unit": "records/s", "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": v, "unit": "records/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def count_launches(step, skip=()):
    """Kernels launched by one (untimed) step, from a CUDA-activity trace: (ours, names).  'Ours' = every
    kernel compiled into libowl.so (fold / tables / KS / exchange kernels and the CUB sort kernels
    instantiated there); torch's own memset/copy activity is not a kernel and is not counted, nor are kernels
    whose names contain one of `skip` (the chunked path's untimed on-device generation: tracegen's og_*
    kernels and the torch ops around them)."""
    import torch
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        step()
        torch.cuda.synchronize()
    names = {}
    for ev in prof.events():
        if getattr(ev, "device_type", None) is not None and str(ev.device_type).endswith("CUDA"):
            n = ev.name
            if n.lower().startswith(("memcpy", "memset")) or any(k in n for k in skip):
                continue
            names[n] = names.get(n, 0) + 1
    return sum(names.values()), names


def e2e_leg(args, p, api, tracegen, dev, stream, n_runs_e2e, my_runs, world=1, rank=0):
    """Same metric through the public C ABI with HOST records: every step stages the runs' records from
    pinned host memory into HBM inside owl_build_adcfg (OWL_SEG_HOST_RECORDS), folds, (at N > 1 exchanges
    cells by owner,) diffs and runs the leak test, whose rows come back to the host (D2H).  The first
    n_runs_e2e of each rank's runs (stated) keep the pinned host footprint bounded."""
    import torch
    import torch.distributed as dist
    ctx = api.Context(dev.index)
    ctx.set_config(channel_order=CHANNEL_MODES[args.channel_mode])
    base_run = 1 << 20  # run ids disjoint from the device-resident leg
    runs_f = [r for r in my_runs if tracegen.run_class(p, r) == 0][: n_runs_e2e // 2]
    runs_r = [r for r in my_runs if tracegen.run_class(p, r) == 1][: n_runs_e2e // 2]
    segs, hold, n_rec = [], [], 0
    for r in runs_f + runs_r:
        for m in tracegen.run_segments(p, r):
            buf, n = tracegen.device_records(p, r, m.seq, device=dev, stream=stream)
            if args.channel_order:
                buf = tracegen.device_interleave(buf, n)
            h = torch.empty(buf.shape, dtype=buf.dtype, pin_memory=True)
            h.copy_(buf)
            del buf
            hold.append(h)
            segs.append(api.Segment(base_run + r, m.input_class, m.seq, m.n_warps, m.kernel_id, h, n,
                                    flags=api.OWL_SEG_HOST_RECORDS | (0 if args.channel_order else api.OWL_SEG_WARP_MAJOR)))
            n_rec += n
    torch.cuda.synchronize()
    ctx.ingest(segs, stream)
    rf = [base_run + r for r in runs_f]
    rr = [base_run + r for r in runs_r]
    if world > 1:
        from paper_conf_dsn_zhaoxcqzj24_b200 import dist as D
        mine = rf + rr
        meta = {base_run + r: (tracegen.run_class(p, r), [m.kernel_id for m in tracegen.run_segments(p, r)])
                for r in runs_f + runs_r}
        allm = D.gather_sequences(meta)
        D.agree_slots(ctx, allm, mine)
        rf = sorted(r for r, (c, _) in allm.items() if c == 0)
        rr = sorted(r for r, (c, _) in allm.items() if c == 1)
    d2h = [0]

    def step():
        ef, er = ctx.build(rf), ctx.build(rr)
        held = [ef, er]
        if world > 1:
            (ef, bf), (er, br) = D.owner_evidence(ctx, ef, world, rank), D.owner_evidence(ctx, er, world, rank)
            held += [ef, er]
            d, lk = D.diff(ctx, ef, er), D.leak_test(ctx, ef, er, 0.05)
        else:
            d, lk = ctx.diff(ef, er), ctx.leak_test(ef, er, 0.05)
        d2h[0] = d.nbytes + lk.nbytes
        for g in held:
            g.destroy()

    for _ in range(max(1, args.warmup)):
        step()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    steps = max(1, min(args.steps, 3))
    e0.record(stream)
    for _ in range(steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    total = n_rec
    if world > 1:
        t = torch.tensor([ms, float(n_rec)], device=dev, dtype=torch.float64)
        mx = t.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        ms, total = float(mx[0].item()), int(t[1].item())
    del ctx, segs, hold
    return {"value": total / (ms / 1e3), "unit": "records/s", "h2d_bytes_per_step": 16 * total,
            "d2h_bytes_per_step": d2h[0], "ms_per_step": ms, "records_per_step": total,
            "sample": f"{len(runs_f)} FIX + {len(runs_r)} RND runs per GPU of the same workload from pinned host "
                      f"memory, {steps} steps"}


def _chunks(tracegen, p, runs, budget_bytes):
    """Contiguous blocks of the (ascending) runs whose records fit in `budget_bytes` of HBM at once (record sizes
    estimated from the first runs; exactness never depends on the split)."""
    if not runs:
        return []
    sample = runs[:2]
    per_run = 16 * sum(tracegen.host_count(p, r, m.seq) for r in sample for m in tracegen.run_segments(p, r)) / len(sample)
    k = max(1, int(budget_bytes // max(per_run, 1.0)))
    return [runs[i:i + k] for i in range(0, len(runs), k)]


def run_ours(args):
    import torch
    import torch.distributed as dist

    import tracegen
    from paper_conf_dsn_zhaoxcqzj24_b200 import api

    world, rank, local = _dist()
    # OWL_BENCH_SHARE_GPU=1 (tests only): ranks share the box's GPUs round-robin and use gloo, so the N > 1
    # path can be exercised on one GPU; the measured configuration is one rank per GPU over NCCL.
    share = os.environ.get("OWL_BENCH_SHARE_GPU") == "1"
    if share:
        local = local % torch.cuda.device_count()
    if world > 1:
        if share:
            dist.init_process_group("gloo")
        else:
            os.environ.setdefault("NCCL_DEBUG", "INFO")  # the driver checks comm_nranks in the log
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cfg = args.config
    base = tracegen.Params.preset(cfg)
    # scaling: weak (default: every rank holds the full per-GPU workload of its own runs) or strong (C5, the north
    # star's scaling sweep: the paper-size run set is split across the ranks)
    strong = args.scaling == "strong" or (args.scaling == "auto" and cfg == 5)
    if strong:
        p = base
        from paper_conf_dsn_zhaoxcqzj24_b200 import dist as D
        my_runs = D.shard(list(range(p.n_runs)), world, rank) if world > 1 else list(range(p.n_runs))
    else:
        rpr = base.n_runs
        p = tracegen.Params.preset(cfg, runs_fix=base.runs_fix * world, runs_rnd=base.runs_rnd * world)
        my_runs = list(range(rank * rpr, (rank + 1) * rpr))
    if args.runs:
        my_runs = my_runs[: args.runs]
    ctx = api.Context(local)
    ctx.set_config(channel_order=CHANNEL_MODES[args.channel_mode])
    stream = torch.cuda.current_stream(dev)
    chunks = _chunks(tracegen, p, my_runs, args.hbm_budget_gb * 1e9)
    resident = len(chunks) == 1
    if not resident and world > 1:
        raise SystemExit("bench: a rank's runs exceed --hbm-budget-gb; use more GPUs or strong scaling")

    def generate(runs):
        segs = []
        for r in runs:
            for m in tracegen.run_segments(p, r):
                buf, n = tracegen.device_records(p, r, m.seq, device=dev, stream=stream)
                if args.channel_order:  # a tracer channel's order (reading R17): bursts of 32, warps round-robin
                    buf = tracegen.device_interleave(buf, n)
                segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, n,
                                        flags=0 if args.channel_order else api.OWL_SEG_WARP_MAJOR))
        torch.cuda.synchronize()
        return segs

    t_gen = time.perf_counter()
    segs = generate(chunks[0]) if chunks else []
    t_gen = time.perf_counter() - t_gen
    n_records = sum(s.n_records for s in segs)
    if not resident:
        for c in chunks[1:]:
            n_records += sum(tracegen.host_count(p, r, m.seq) for r in c for m in tracegen.run_segments(p, r))
    ctx.ingest(segs, stream)
    if world > 1:
        # §8(e): slot agreement over all runs, then every step folds this rank's shard into partial evidences
        # and exchanges cells by owner (paper_conf_dsn_zhaoxcqzj24_b200/dist.py)
        from paper_conf_dsn_zhaoxcqzj24_b200 import dist as D
        meta = {r: (tracegen.run_class(p, r), [m.kernel_id for m in tracegen.run_segments(p, r)]) for r in my_runs}
        all_meta = D.gather_sequences(meta)
        D.agree_slots(ctx, all_meta, my_runs)
        all_runs = sorted(all_meta)
    else:
        all_runs = list(my_runs)
    rf_all, rr_all = _class_runs(p, all_runs, 0), _class_runs(p, all_runs, 1)

    out = {}
    brk = {}
    timed_ms = [0.0]

    def tick(name, t0):
        if args.breakdown:
            torch.cuda.synchronize()
            t1 = time.perf_counter()
            brk[name] = brk.get(name, 0.0) + (t1 - t0) * 1e3
            return t1
        return t0

    def analysis(ef, er, held):
        t0 = time.perf_counter()
        if world > 1:  # the one exchange: partial evidences -> owners' evidences
            (ef, bf), (er, br) = D.owner_evidence(ctx, ef, world, rank), D.owner_evidence(ctx, er, world, rank)
            held += [ef, er]
            t0 = tick("exchange", t0)
            d = D.diff(ctx, ef, er)
            t0 = tick("diff", t0)
            lk = D.leak_test(ctx, ef, er, 0.05)
        else:
            d = ctx.diff(ef, er)
            t0 = tick("diff", t0)
            lk = ctx.leak_test(ef, er, 0.05)
        tick("leak_test", t0)
        out.update(n_diff=len(d), n_leaks=len(lk), info_f=ef.info(), info_r=er.info())
        if args.dump:
            out.update(diff_rows=np.array(d), leak_rows=np.array(lk))

    def step():
        if resident:
            t0 = time.perf_counter()
            ef = ctx.build(rf_all)
            t0 = tick("build_fix", t0)
            er = ctx.build(rr_all)
            tick("build_rnd", t0)
            held = [ef, er]
            analysis(ef, er, held)
            for g in held:
                g.destroy()
            return
        # chunked (the workload exceeds one GPU's HBM): each chunk's records are generated (untimed), then
        # folded and merged into the evidences (timed, CUDA events); the analysis is timed
        nonlocal segs
        ev = {0: None, 1: None}
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for ci, c in enumerate(chunks):
            if ci > 0 or segs is None:
                ctx.forget_runs([r for r in my_runs if r not in c])
                segs = None
                torch.cuda.empty_cache()
                segs = generate(c)
                ctx.ingest(segs, stream)
            e0.record(stream)
            cset = set(c)
            for cls, allc in ((0, rf_all), (1, rr_all)):
                mine = [r for r in allc if r in cset]
                if not mine:
                    continue
                if ev[cls] is None:
                    ev[cls] = ctx.build(mine)
                else:
                    ev[cls].accumulate(mine)
            e1.record(stream)
            torch.cuda.synchronize()
            timed_ms[0] += e0.elapsed_time(e1)
        e0.record(stream)
        held = [ev[0], ev[1]]
        analysis(ev[0], ev[1], held)
        e1.record(stream)
        torch.cuda.synchronize()
        timed_ms[0] += e0.elapsed_time(e1)
        for g in held:
            g.destroy()
        # the next step starts from the first chunk again
        ctx.forget_runs(my_runs)
        segs = None
        torch.cuda.empty_cache()
        segs = generate(chunks[0])
        ctx.ingest(segs, stream)

    clocks = ClockSampler(local)
    clocks.start()  # nvidia-smi starts up during the warm-up; only timed-region samples are kept
    for _ in range(args.warmup):
        step()
    brk.clear()
    ctx.reset_stats()
    timed_ms[0] = 0.0
    clocks.wait_ready()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.window = True
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    ck = clocks.stop()
    ms = (e0.elapsed_time(e1) if resident else timed_ms[0]) / args.steps
    st = ctx.stats()
    if world > 1:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
        t = torch.tensor([float(n_records)], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        total_records = int(t.item())
    else:
        total_records = n_records
    value = total_records / (ms / 1e3)
    peak, peak_src = _peaks()
    fold_ms = st["total_fold_ms"] / max(1, st["fold_launches"])
    fold_bytes = 16.0 * st["total_fold_records"] / max(1, st["fold_launches"])
    achieved = fold_bytes / (fold_ms / 1e3) / 1e9
    mode = "strong" if strong else "weak"
    res = {
        "metric": METRIC, "value": value, "unit": "records/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": mode,
        "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": tracegen.CONFIG_NAMES[cfg] + (" (channel order)" if args.channel_order else ""),
                   "record_order": ("channel (bursts of 32, warps round-robin; %s)" % args.channel_mode)
                   if args.channel_order else "warp-major",
                   "runs_per_gpu": len(my_runs), "runs_total": p.n_runs,
                   "records_per_gpu": n_records, "bytes_per_gpu": 16 * n_records,
                   "l2": "inputs (%.1f GB) >> 126 MB L2; no flush needed" % (16 * n_records / 1e9),
                   "parallelism": f"dp{world} (runs sharded, key-hash exchange, {mode} scaling)" if world > 1
                   else "single GPU",
                   "hbm_chunks": len(chunks),
                   "timing": "whole steps, CUDA events" if resident else
                   f"{len(chunks)} chunks per step: each chunk's on-device generation untimed, its fold + merge and "
                   "the analysis timed with CUDA events",
                   "generate_s_untimed": round(t_gen, 2)},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": _traffic(fold_bytes / 16.0) if cfg == 2 else None, "kernel": "fold_kernel",
                     "note": f"16 B/record algorithmic; {st['fold_launches']} fold launches, "
                             f"{fold_ms:.2f} ms avg (CUDA events on the launch stream); peak {peak_src}"},
        "clocks": ck,
        "fold_share_of_step": (st["total_fold_ms"] / args.steps) / ms,
        "breakdown_ms": {k: v / args.steps for k, v in brk.items()} if args.breakdown else None,
        "result": {"n_diff_rows": out.get("n_diff"), "n_leaks": out.get("n_leaks"),
                   "cells_fix": out.get("info_f", {}).get("n_cells"), "cells_rnd": out.get("info_r", {}).get("n_cells")},
    }
    n_launch, names = count_launches(step, () if resident else ("og_", "at::", "native::", "at_cuda_detail"))
    res["gpu_launches"] = n_launch * args.steps
    res["gpu_launches_per_step"] = names
    if not args.no_e2e:
        del segs
        ctx.forget_runs(my_runs)
        torch.cuda.empty_cache()
        per_run = 16 * n_records / max(1, len(my_runs))
        e2e_runs = max(2, min(args.e2e_runs, int(args.e2e_gb * 1e9 // max(per_run, 1)) // 2 * 2))
        res["e2e"] = e2e_leg(args, p, api, tracegen, dev, stream, e2e_runs, my_runs, world, rank)
    if rank == 0 and not args.no_cpu:
        res["cpu_baseline"] = cpu_baseline(cfg, args.cpu_seconds)
    if rank == 0 and args.dump:  # the last step's result rows (tests: the N > 1 path against the oracle)
        os.makedirs(args.dump, exist_ok=True)
        np.save(os.path.join(args.dump, "diff.npy"), out["diff_rows"])
        np.save(os.path.join(args.dump, "leaks.npy"), out["leak_rows"])
        with open(os.path.join(args.dump, "runs.json"), "w") as f:
            json.dump({"config": cfg, "runs_fix": p.runs_fix, "runs_rnd": p.runs_rnd, "runs": all_runs}, f)
    if rank == 0:
        print(json.dumps(res), flush=True)
    if world > 1:
        dist.destroy_process_group()


CHANNEL_MODES = {"auto": 0, "copy": 1, "inplace": 2}  # owl_config.channel_order (auto = in place)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", type=int, default=2, help="workload C1..C5 (default: configs[1], C2)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--runs", type=int, default=0, help="limit runs per GPU (debug)")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-runs", type=int, default=20, help="runs (half FIX, half RND) in the host-records e2e leg")
    ap.add_argument("--breakdown", action="store_true", help="host-timed per-call breakdown (syncs between calls)")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--scaling", default="auto", choices=["auto", "weak", "strong"],
                    help="auto: strong for C5 (the scaling sweep: 1000 runs split across the ranks), weak otherwise")
    ap.add_argument("--hbm-budget-gb", type=float, default=140.0, help="records resident at once per GPU")
    ap.add_argument("--e2e-gb", type=float, default=8.0, help="pinned host bytes of the e2e leg's runs (bound)")
    ap.add_argument("--channel-order", action="store_true",
                    help="records in a tracer channel's order (bursts of 32 per warp, warps round-robin; N2)")
    ap.add_argument("--channel-mode", default="auto", choices=sorted(CHANNEL_MODES),
                    help="channel-order bucketing: copy to warp-major, fold in place, or auto (owl_config.channel_order)")
    ap.add_argument("--dump", default="", help="rank 0 writes the last step's diff / leak rows here (tests)")
    args = ap.parse_args()
    import __graft_entry__
    __graft_entry__.build_native()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
