"""Shared helpers of the GPU parity tests: segment construction for both sides and the parity bar
(BASELINE.json north_star): canonical dumps and diff rows bit-exact, K exact, D bit-identical,
p within 1e-9 relative (x when p underflows), verdicts identical except within 1e-9 of the threshold."""
import math

import numpy as np
import torch

import tracegen
from oracle import oracle
from paper_conf_dsn_zhaoxcqzj24_b200 import api
from tests import helpers as H

SIG = 0.05


def _gpu_segments(p, runs, interleaved=False):
    segs = []
    for r in runs:
        for m in tracegen.run_segments(p, r):
            if interleaved:
                rec = tracegen.interleave(tracegen.host_records(p, r, m.seq))
                buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
                segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, len(rec), flags=0))
            else:
                buf, n = tracegen.device_records(p, r, m.seq)
                segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, n))
    return segs


def _oracle_segments(p, runs):
    out = {0: [], 1: []}
    for r in runs:
        for m in tracegen.run_segments(p, r):
            out[m.input_class].append(oracle.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id,
                                                     tracegen.host_records(p, r, m.seq)))
    return out


def _runs_of(p, cls):
    return [r for r in range(p.n_runs) if tracegen.run_class(p, r) == cls]


def _same_p(a, b):
    if a == b:
        return True
    if a < 2.2250738585072014e-308 or b < 2.2250738585072014e-308:
        xa, xb = -math.log(max(a, 5e-324) / 2), -math.log(max(b, 5e-324) / 2)
        return abs(xa - xb) <= 1e-9 * max(abs(xa), abs(xb)) or (a == 0 and b == 0)
    return abs(a - b) <= 1e-9 * max(abs(a), abs(b))


def assert_ks_parity(g, o):
    assert len(g) == len(o)
    for f in ("kind", "slot_fix", "slot_rnd", "bb", "ins", "j", "n", "m", "K_lo", "K_hi"):
        assert np.array_equal(g[f], o[f]), f
    assert np.array_equal(g["D"].view(np.uint64), o["D"].view(np.uint64)), "D must be bit-identical"
    for i in range(len(g)):
        assert _same_p(float(g["p"][i]), float(o["p"][i])), (i, g["p"][i], o["p"][i])
        if g["fail"][i] != o["fail"][i]:
            assert abs(float(o["p"][i]) - SIG) <= 1e-9 * SIG, i


def assert_leak_parity(g, o):
    near = [i for i in range(len(o)) if o["kind"][i] != 0 and abs(float(o["p"][i]) - SIG) <= 1e-9 * SIG]
    assert not near, "a p-value inside the tolerance band of the threshold: compare verdicts by hand"
    assert len(g) == len(o)
    for f in ("kind", "slot_fix", "slot_rnd", "bb", "ins", "j", "kernel_id", "n", "m", "K_lo", "K_hi"):
        assert np.array_equal(g[f], o[f]), f
    ks = g["kind"] != 0
    assert np.array_equal(g["D"][ks].view(np.uint64), o["D"][ks].view(np.uint64))
    for i in np.flatnonzero(ks):
        assert _same_p(float(g["p"][i]), float(o["p"][i]))


def _build_and_compare(ctx, p, runs=None, interleaved=False):
    runs = list(range(p.n_runs)) if runs is None else runs
    segs = _gpu_segments(p, runs, interleaved)
    ctx.ingest(segs)
    try:
        rf = [r for r in runs if tracegen.run_class(p, r) == 0]
        rr = [r for r in runs if tracegen.run_class(p, r) == 1]
        ef, er = ctx.build(rf), ctx.build(rr)
        osg = _oracle_segments(p, runs)
        of, orr = oracle.build(osg[0]), oracle.build(osg[1])
        bf, bo = ef.export(), of.export()
        if bf != bo:
            pf, po = H.parse_blob(bf), H.parse_blob(bo)
            for t in ("slots", "node", "edge", "triple", "addr"):
                assert len(pf[t]) == len(po[t]) and np.array_equal(pf[t], po[t]), t
        assert bf == bo
        assert er.export() == orr.export()
        assert_ks_parity(ctx.ks_tests(ef, er, SIG), oracle.ks_tests(of, orr, SIG))
        assert_leak_parity(ctx.leak_test(ef, er, SIG), oracle.leak_test(of, orr, SIG))
        gd, od = ctx.diff(ef, er), oracle.diff(of, orr)
        assert len(gd) == len(od) and np.array_equal(gd, od)
        return ef, er, of, orr
    finally:
        ctx.forget_runs(runs)
