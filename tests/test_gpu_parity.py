"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded inputs.

Bar (BASELINE.json north_star): canonical A-DCFG dumps (node / edge / triple / address tables,
slot table) and diff rows bit-exact; KS K exact and D bit-identical; p within 1e-9 relative (x when p underflows);
leak verdicts and locations identical except where p is within 1e-9 of the threshold.
"""
import numpy as np
import pytest

import tracegen
from oracle import oracle
from tests import helpers as H

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_dsn_zhaoxcqzj24_b200 import api  # noqa: E402
from tests.gpu_common import (SIG, _build_and_compare, _gpu_segments, _oracle_segments, _runs_of,  # noqa: E402
                              assert_ks_parity, assert_leak_parity)


@pytest.fixture(scope="module")
def ctx():
    return api.Context(0)


def test_generator_device_equals_host():
    """T3: the counter-based generator gives byte-identical records on host and device."""
    for cfg, div in ((1, 1), (2, 64), (3, 16), (4, 128), (5, 32), (9, 16)):
        p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=1, runs_rnd=1)
        for r in (0, 1):
            for m in tracegen.run_segments(p, r):
                buf, n = tracegen.device_records(p, r, m.seq)
                host = tracegen.host_records(p, r, m.seq)
                assert n == len(host)
                assert bytes(buf.cpu().numpy()) == host.tobytes(), (cfg, r, m.seq)
    for cfg, t in ((6, 1000), (7, 333), (8, 50)):
        p = tracegen.Params.preset(cfg, threads=t)
        for m in tracegen.run_segments(p, 0):
            buf, n = tracegen.device_records(p, 0, m.seq)
            assert bytes(buf.cpu().numpy()) == tracegen.host_records(p, 0, m.seq).tobytes(), cfg


def test_w1(ctx):
    doc = H.load_golden("w1.json")
    rec = H.w1_records(doc)
    buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
    ctx.ingest([api.Segment(0, 0, 0, 2, 10, buf, len(rec))])
    try:
        g = ctx.build([0])
        p = H.parse_blob(g.export())
        got = H.blob_tables_as_lists(p)
        for t in ("node", "edge", "triple", "addr"):
            assert got[t] == doc["expected"][t], t
        assert g.export() == oracle.build([oracle.Segment(0, 0, 0, 2, 10, rec)]).export()
    finally:
        ctx.forget_runs([0])


@pytest.mark.parametrize("variant", ["mem_before_bb", "bb_mismatch", "gwarp", "bb_fields", "mtype"])
def test_malformed_same_report(ctx, variant):
    rec = H.w1_records()
    if variant == "mem_before_bb":
        rec = np.concatenate([rec[1:2], rec[0:1], rec[2:]])
    elif variant == "bb_mismatch":
        rec["meta"][4] = (rec["meta"][4] & ~np.uint32(0x3FFFF << 8)) | np.uint32(2 << 8)
    elif variant == "gwarp":
        rec["gwarp"][10:] = 7
    elif variant == "bb_fields":
        rec["addr"][3] = 5
    else:
        rec["addr"][7] = np.uint64(12) << np.uint64(60)
    with pytest.raises(oracle.OracleError) as eo:
        oracle.build([oracle.Segment(0, 0, 0, 2, 10, rec)])
    buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
    # warp-major, then channel order with the bursts copied to warp-major order and folded in place
    for flags, mode in ((api.OWL_SEG_WARP_MAJOR, 0), (0, api.OWL_CHANNEL_COPY), (0, api.OWL_CHANNEL_IN_PLACE)):
        ctx.set_config(channel_order=mode)
        ctx.ingest([api.Segment(0, 0, 0, 2, 10, buf, len(rec), flags=flags)])
        try:
            with pytest.raises(api.OwlError, match="OWL_ERR_MALFORMED_TRACE") as eg:
                ctx.build([0])
            assert str(eo.value).split(": ", 1)[1] in str(eg.value), (str(eo.value), str(eg.value))
        finally:
            ctx.forget_runs([0])
            ctx.set_config()


@pytest.mark.parametrize("cfg,div,nf,nr", [(1, 1, 10, 10), (2, 32, 3, 3), (3, 16, 2, 2), (4, 64, 2, 2), (5, 16, 3, 3)])
def test_config_parity(ctx, cfg, div, nf, nr):
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=nf, runs_rnd=nr)
    _build_and_compare(ctx, p)


def test_c4_kernel_leak_parity(ctx):
    """C4 at small scale with enough RND runs that some skip the conditional kernel (Myers inserts)."""
    p = tracegen.Params.preset(4, grid_div=256, runs_fix=3, runs_rnd=6)
    ef, er, of, orr = _build_and_compare(ctx, p)
    assert ef.info()["n_slots"] == 4


@pytest.mark.parametrize("mode", [api.OWL_CHANNEL_COPY, api.OWL_CHANNEL_IN_PLACE])
@pytest.mark.parametrize("cfg,div", [(1, 1), (2, 64), (5, 32)])
def test_channel_order_input(ctx, cfg, div, mode):
    """Reading R17: interleaved (channel-order) records give the identical A-DCFG, whether the bursts are copied
    to warp-major order or folded in place through the burst index (owl_config.channel_order)."""
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=2, runs_rnd=2)
    ctx.set_config(channel_order=mode)
    try:
        _build_and_compare(ctx, p, interleaved=True)
    finally:
        ctx.set_config()


def test_accumulate_equals_single_build(ctx):
    p = tracegen.Params.preset(4, grid_div=256, runs_fix=4, runs_rnd=4)
    runs = list(range(p.n_runs))
    ctx.ingest(_gpu_segments(p, runs))
    try:
        rr = _runs_of(p, 1)
        whole = ctx.build(rr)
        part = ctx.build(rr[:2])
        part.accumulate(rr[2:])
        assert part.export() == whole.export()
        with pytest.raises(api.OwlError, match="INVALID_ARG"):
            part.accumulate(rr[:1])  # runs must be merged in ascending order
    finally:
        ctx.forget_runs(runs)


def test_identical_inputs_no_differences(ctx):
    """North-star invariant: identical traces => zero diff rows, every D = 0, no leaks."""
    p = tracegen.Params.preset(2, grid_div=64, runs_fix=3, runs_rnd=1)
    runs = _runs_of(p, 0)
    ctx.ingest(_gpu_segments(p, runs))
    try:
        a, b = ctx.build(runs), ctx.build(runs)
        assert len(ctx.diff(a, b)) == 0
        ks = ctx.ks_tests(a, b)
        assert len(ks) > 0 and np.all(ks["D"] == 0.0) and np.all(ks["p"] == 2.0)
        assert len(ctx.leak_test(a, b)) == 0
        r0, r1 = ctx.build(runs[:1]), ctx.build(runs[1:2])  # FIX runs repeat one secret
        assert len(ctx.diff(r0, r1)) == 0
    finally:
        ctx.forget_runs(runs)


def test_capacity_regrow(ctx):
    """A deliberately tiny initial table must regrow and still give the exact result."""
    p = tracegen.Params.preset(2, grid_div=64, runs_fix=1, runs_rnd=1)
    ctx.set_config(addr_capacity=1024, cf_capacity=16)
    try:
        _build_and_compare(ctx, p)
    finally:
        ctx.set_config()


def test_full_size_c2_run_parity(ctx):
    """configs[1] (C2, the bench workload) at full size in the bench's launch configuration: one run's
    A-DCFG against the oracle, and E_fix over 4 FIX runs = 4 x that run (FIX repeats one secret)."""
    p = tracegen.Params.preset(2, runs_fix=4, runs_rnd=0)
    segs = _gpu_segments(p, [0, 1, 2, 3])
    ctx.ingest(segs)
    try:
        g0 = ctx.build([0])
        o0 = oracle.build(_oracle_segments(p, [0])[0])
        assert g0.export() == o0.export()
        ev = H.parse_blob(ctx.build([0, 1, 2, 3]).export())
        one = H.parse_blob(g0.export())
        for t in ("node", "edge", "triple", "addr"):
            assert np.array_equal(ev[t]["count"], 4 * one[t]["count"]), t
        n_rec = sum(s.n_records for s in segs)
        assert int(ev["addr"]["count"].sum()) + int(ev["node"]["count"].sum()) == n_rec
    finally:
        ctx.forget_runs([0, 1, 2, 3])


def test_work_queue_stress_long_warps(ctx):
    """C3 traced warps (~107K records) span many tiles, so most tiles hold no warp start and warps re-pop the
    CTA queue immediately; 40 identical FIX runs must give exactly 40 x one run (a duplicated or skipped
    tile would break it), and one run must match the oracle."""
    p = tracegen.Params.preset(3, grid_div=16, runs_fix=40, runs_rnd=0)
    runs = list(range(40))
    ctx.ingest(_gpu_segments(p, runs))
    try:
        one = ctx.build([0])
        assert one.export() == oracle.build(_oracle_segments(p, [0])[0]).export()
        ev, o = H.parse_blob(ctx.build(runs).export()), H.parse_blob(one.export())
        for t in ("node", "edge", "triple", "addr"):
            assert np.array_equal(ev[t]["count"], 40 * o[t]["count"]), t
    finally:
        ctx.forget_runs(runs)


def _build_one(ctx, rec, n_warps, flags=None):
    buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
    seg = api.Segment(0, 0, 0, n_warps, 10, buf, len(rec)) if flags is None else \
        api.Segment(0, 0, 0, n_warps, 10, buf, len(rec), flags=flags)
    ctx.ingest([seg])
    try:
        return ctx.build([0]).export()
    finally:
        ctx.forget_runs([0])


@pytest.mark.parametrize("seed", range(12))
def test_random_traces_parity(ctx, seed):
    """Random valid traces (random active-lane subsets, so chunks straddle instructions; small address pools,
    so broadcast / window / scattered chunks mix; repeated BBs): GPU = oracle, warp-major and interleaved."""
    rng = np.random.default_rng(1000 + seed)
    n_warps = int(rng.integers(1, 40))
    rec = H.random_trace(rng, n_warps=n_warps, max_bbs=int(rng.integers(1, 30)), n_bb_ids=int(rng.integers(1, 12)),
                         max_ins=int(rng.integers(1, 6)), n_addr=int(rng.integers(1, 600)),
                         active=float(rng.uniform(0.3, 1.0)))
    if len(rec) == 0:
        return
    want = oracle.build([oracle.Segment(0, 0, 0, n_warps, 10, rec)]).export()
    assert _build_one(ctx, rec, n_warps) == want
    inter = H.interleave_random(rng, rec)
    for mode in (api.OWL_CHANNEL_COPY, api.OWL_CHANNEL_IN_PLACE):
        ctx.set_config(channel_order=mode)
        try:
            assert _build_one(ctx, inter, n_warps, flags=0) == want
        finally:
            ctx.set_config()


def test_many_distinct_bbs(ctx):
    """Traced warps visiting up to 700 distinct BBs (beyond the 32 held in registers: the overflow visit map),
    several times each, so j counts per BB; one more distinct BB than the fold supports is a capacity error."""
    rng = np.random.default_rng(7)
    rows = []
    for w in range(6):
        bbs = rng.permutation(5000)[: 100 * (w + 1) + 1]
        for rep in range(3):
            for b in bbs:
                rows.append(H.bb_rec(w, int(b)))
                for lane in range(0, 32, 3):
                    rows.append(H.mem_rec(w, int(b), rep, lane, (3 << 60) | int(rng.integers(0, 64)) * 4))
    rec = H.to_records(rows)
    want = oracle.build([oracle.Segment(0, 0, 0, 6, 10, rec)]).export()
    assert _build_one(ctx, rec, 6) == want
    limit = 32 + 1024  # register visit map + overflow map (owl_fold.cu VCAP; DESIGN.md §5 limits)
    over = H.to_records([H.bb_rec(0, b) for b in range(limit + 1)])
    with pytest.raises(api.OwlError, match="OWL_ERR_CAPACITY"):
        _build_one(ctx, over, 1)


@pytest.mark.parametrize("n_nodes", [1, 3, 4095, 4096, 4097, 5000])
def test_small_table_sort_boundary(ctx, n_nodes):
    """Tables of at most 4096 cells are sorted by one CTA (bitonic in shared memory), larger ones by CUB: node /
    edge / triple tables of sizes around the switch (distinct BB chains split over warps of <= 1000 BBs each)
    export the oracle's canonical order."""
    rows, b, left, w = [], 0, n_nodes, 0
    while left:
        k = min(left, 1000)
        rows += [H.bb_rec(w, b + i) for i in range(k)]
        b, left, w = b + k, left - k, w + 1
    rec = H.to_records(rows)
    want = oracle.build([oracle.Segment(0, 0, 0, w, 10, rec)]).export()
    assert _build_one(ctx, rec, w) == want


def test_wide_keys_sort_fallback(ctx):
    """More than 64 key bits vary across the address table (random 60-bit addresses, every ins and many j):
    the canonical sort takes the full 128-bit path; tables and diff still match the oracle."""
    rng = np.random.default_rng(11)
    rows = []
    for w in range(8):
        for v in range(40):
            b = int(rng.integers(0, 3))
            rows.append(H.bb_rec(w, b))
            for ins in range(int(rng.integers(1, 4))):
                i = int(rng.integers(0, 256))
                for lane in range(32):
                    x = (int(rng.integers(0, 9)) << 60) | int(rng.integers(0, 1 << 60))
                    rows.append(H.mem_rec(w, b, i, lane, x))
    rec = H.to_records(rows)
    of = oracle.build([oracle.Segment(0, 0, 0, 8, 10, rec)])
    assert _build_one(ctx, rec, 8) == of.export()
    assert H.parse_blob(of.export())["addr"].shape[0] > 4096


@pytest.mark.parametrize("cfg,div,nf,nr", [(1, 1, 3, 3), (2, 64, 3, 3), (4, 256, 2, 3), (5, 32, 2, 2)])
def test_filter_inputs_parity(ctx, cfg, div, nf, nr):
    """N1: the GPU partition of runs into classes of identical traces equals the oracle's."""
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=nf, runs_rnd=nr)
    runs = list(range(p.n_runs))
    ctx.ingest(_gpu_segments(p, runs))
    try:
        order = runs[::-1]  # visiting order decides the class ids
        gc, gn = ctx.filter_inputs(order)
        by_run = [(r, [oracle.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, tracegen.host_records(p, r, m.seq))
                       for m in tracegen.run_segments(p, r)]) for r in order]
        oc, on = oracle.filter_inputs(by_run)
        assert gn == on and list(gc) == oc
    finally:
        ctx.forget_runs(runs)


def test_filter_inputs_copies_and_changed_record(ctx):
    rec = H.w1_records()
    other = rec.copy()
    i = int(np.flatnonzero(other["meta"] >> 31)[-1])
    other["addr"][i] = other["addr"][i] + np.uint64(4)
    bufs = [torch.from_numpy(x.view(np.uint8).copy()).cuda() for x in (rec, rec, other, rec)]
    ctx.ingest([api.Segment(r, r % 2, 0, 2, 10, b, len(rec)) for r, b in enumerate(bufs)])
    try:
        cls, n = ctx.filter_inputs([0, 1, 2, 3])
        assert list(cls) == [0, 0, 1, 0] and n == 2
        with pytest.raises(api.OwlError, match="INVALID_ARG"):
            ctx.filter_inputs([0, 0])
    finally:
        ctx.forget_runs([0, 1, 2, 3])


@pytest.mark.parametrize("cfg,threads", [(6, 100), (6, 3000), (7, 1000), (8, 10)])
def test_rq2_workloads_parity(ctx, cfg, threads):
    """N4: the RQ2 trace-size workloads (partial last warps included) fold bit-exactly."""
    p = tracegen.Params.preset(cfg, threads=threads, runs_fix=1, runs_rnd=1)
    _build_and_compare(ctx, p)


@pytest.mark.parametrize("cfg,div,nf,nr", [(2, 64, 3, 3), (4, 256, 2, 3), (9, 8, 3, 5)])
def test_sharded_exchange_equals_one_gpu(cfg, div, nf, nr):
    """§8(e) on one GPU: two 'ranks' (two contexts) each fold a shard of the runs with agreed slots, partition
    their partial evidences by owner, the buckets are exchanged (the all-to-all, done by hand), and each owner
    absorbs its cells: the owners' leak rows, KS rows and diff rows, merged, equal the oracle's on all runs."""
    from paper_conf_dsn_zhaoxcqzj24_b200 import dist as D
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=nf, runs_rnd=nr)
    runs = list(range(p.n_runs))
    world = 2
    ctxs = [api.Context(0) for _ in range(world)]
    keep = []
    meta = {r: (tracegen.run_class(p, r), [m.kernel_id for m in tracegen.run_segments(p, r)]) for r in runs}
    parts = {}
    for rank, c in enumerate(ctxs):
        mine = D.shard(runs, world, rank)
        segs = _gpu_segments(p, mine)
        keep.append(segs)
        c.ingest(segs)
        D.agree_slots(c, meta, mine)
        for cls in (0, 1):
            parts[(rank, cls)] = c.build([r for r in runs if tracegen.run_class(p, r) == cls])
    owned = {}
    for cls in (0, 1):
        bufs = []
        for rank in range(world):
            ptr, sb = parts[(rank, cls)].partition(world)
            whole = torch.as_tensor(D._DeviceBytes(ptr, sum(sb)), device="cuda") if sum(sb) else \
                torch.empty(0, dtype=torch.uint8, device="cuda")
            bufs.append((whole.clone(), sb))
        for owner in range(world):
            pieces, rb = [], []
            for rank in range(world):
                whole, sb = bufs[rank]
                off = sum(sb[:owner])
                pieces.append(whole[off: off + sb[owner]])
                rb.append(sb[owner])
            recv = torch.cat(pieces)
            keep.append(recv)
            owned[(owner, cls)] = ctxs[owner].absorb(parts[(owner, cls)], recv.data_ptr() if recv.numel() else None,
                                                     rb, owner)
    leaks = ctxs[0].merge_leaks(owned[(0, 0)], owned[(0, 1)],
                                [ctxs[o].leak_test(owned[(o, 0)], owned[(o, 1)], SIG) for o in range(world)])
    diffs = ctxs[0].merge_diffs(owned[(0, 0)], owned[(0, 1)],
                                [ctxs[o].diff(owned[(o, 0)], owned[(o, 1)]) for o in range(world)])
    ks = np.concatenate([ctxs[o].ks_tests(owned[(o, 0)], owned[(o, 1)], SIG) for o in range(world)])
    osg = _oracle_segments(p, runs)
    of, orr = oracle.build(osg[0]), oracle.build(osg[1])
    assert_leak_parity(leaks, oracle.leak_test(of, orr, SIG))
    od = oracle.diff(of, orr)
    assert len(diffs) == len(od) and np.array_equal(diffs, od)
    oks = oracle.ks_tests(of, orr, SIG)
    key = lambda a: np.lexsort((a["j"], a["ins"], a["bb"], a["slot_fix"], a["kind"]))  # noqa: E731
    assert_ks_parity(ks[key(ks)], oks[key(oks)])
    for c in ctxs:  # owners test their own nodes under R2 as well (each node's cells live on one owner)
        c.set_config(hcf_reading=1)
    ks2 = np.concatenate([ctxs[o].ks_tests(owned[(o, 0)], owned[(o, 1)], SIG) for o in range(world)])
    ks2 = ks2[key(ks2)]
    oks = oks[key(oks)]
    for f in ("kind", "slot_fix", "slot_rnd", "bb", "ins", "j", "n", "m"):
        assert np.array_equal(ks2[f], oks[f]), f
    _assert_r2_rows(ks2, oks, of, orr)


# ---- N3: H_cf reading R2 (row-normalized transition matrix A, Eqs. 7-8) -------------------------------
def _r2_oracle_rows(of, orr, o_ks):
    """R2 statistic for every CF pair the oracle tests (same pairs as R1: node present on both aligned sides)."""
    from oracle import hcf_r2
    tf, tr = H.parse_blob(of.export())["triple"], H.parse_blob(orr.export())["triple"]
    out = []
    for row in o_ks[o_ks["kind"] == 1]:
        cf = hcf_r2.node_cells(tf, int(row["slot_fix"]), int(row["bb"]))
        cr = hcf_r2.node_cells(tr, int(row["slot_rnd"]), int(row["bb"]))
        out.append(hcf_r2.ks_r2(cf, cr, SIG))
    return out


def _assert_r2_rows(g_ks, o_ks, of, orr):
    """GPU KS rows under R2 (same order as the oracle's R1 rows) against the rational R2 oracle; returns the
    (slot_fix, bb) of the failing CF rows."""
    cf = np.flatnonzero(g_ks["kind"] == 1)
    r2 = _r2_oracle_rows(of, orr, o_ks)
    assert len(r2) == len(cf) and len(cf) > 0
    fails = set()
    for i, (n, m, D, Dd, po, fo) in zip(cf, r2):
        g = g_ks[i]
        assert int(g["K_lo"]) == 0 and int(g["K_hi"]) == 0
        Dg = float(g["D"])
        assert abs(Dg - float(D)) <= 1e-12, (i, Dg, D)
        w = n * m / (n + m)
        band = 4.0 * Dd * w * 1e-12 + 1e-12
        pg = float(g["p"])
        assert abs(pg - po) <= band * max(po, pg) or (po == 0.0 and pg < 1e-300), (i, pg, po)
        if bool(g["fail"]) != fo:
            assert abs(po - SIG) <= band * SIG, (i, pg, po)
        if g["fail"]:
            fails.add((int(g["slot_fix"]), int(g["bb"])))
    return fails


@pytest.mark.parametrize("cfg,div,nf,nr", [(1, 1, 10, 10), (2, 32, 3, 3), (3, 16, 2, 2), (4, 64, 2, 2),
                                        (5, 16, 3, 3)])
def test_hcf_r2_parity(ctx, cfg, div, nf, nr):
    """Bar for R2: n, m exact; K = 0; |D - D_exact| <= 1e-12 (D is a rational evaluated in fp64
    on the GPU, exactly on the oracle); p within the band that D tolerance implies through Eq. 4
    (|dp/p| <= 4 D w |dD| + 1e-12); verdicts identical outside that band; DF rows identical to R1's."""
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=nf, runs_rnd=nr)
    runs = list(range(p.n_runs))
    ctx.ingest(_gpu_segments(p, runs))
    try:
        ef, er = ctx.build(_runs_of(p, 0)), ctx.build(_runs_of(p, 1))
        osg = _oracle_segments(p, runs)
        of, orr = oracle.build(osg[0]), oracle.build(osg[1])
        o_ks = oracle.ks_tests(of, orr, SIG)
        ctx.set_config(hcf_reading=1)
        try:
            g_ks = ctx.ks_tests(ef, er, SIG)
            g_leaks = ctx.leak_test(ef, er, SIG)
        finally:
            ctx.set_config()
        assert len(g_ks) == len(o_ks)
        for f in ("kind", "slot_fix", "slot_rnd", "bb", "ins", "j", "n", "m"):
            assert np.array_equal(g_ks[f], o_ks[f]), f
        df = g_ks["kind"] == 2
        assert_ks_parity(g_ks[df], o_ks[df])
        fails = _assert_r2_rows(g_ks, o_ks, of, orr)
        g_cf = {(int(r["slot_fix"]), int(r["bb"])) for r in g_leaks if r["kind"] == 1}
        assert g_cf == fails
        o_leaks = oracle.leak_test(of, orr, SIG)
        keep_g, keep_o = g_leaks["kind"] != 1, o_leaks["kind"] != 1  # kernel / DF leaks: independent of H_cf
        assert_leak_parity(g_leaks[keep_g], o_leaks[keep_o])
    finally:
        ctx.forget_runs(runs)


def test_hcf_reading_invalid(ctx):
    with pytest.raises(api.OwlError, match="OWL_ERR_INVALID_ARG"):
        ctx.set_config(hcf_reading=2)
    ctx.set_config()


def test_channel_order_mode_invalid(ctx):
    with pytest.raises(api.OwlError, match="OWL_ERR_INVALID_ARG"):
        ctx.set_config(channel_order=3)
    ctx.set_config()


_MISFLAG_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import tracegen
from tests import helpers as H
from paper_conf_dsn_zhaoxcqzj24_b200 import api
p = tracegen.Params.preset(2, grid_div=16, runs_fix=1, runs_rnd=0)
rec = tracegen.host_records(p, 0, 0)
variants = {{"interleaved": tracegen.interleave(rec)}}
g = rec["gwarp"]
b1, b2, b3 = (int(np.flatnonzero(g == w)[0]) for w in (1, 2, 3))
mid = (b1 + b2) // 2  # warp 2's block moved into the middle of warp 1's (warp 1 then starts twice)
variants["split_warp"] = np.concatenate([rec[:mid], rec[b2:b3], rec[mid:b2], rec[b3:]])
# 100 records of the last warp hidden 50 records past a fold-tile boundary (2^15) inside another warp's block:
# closer than the tile search's sample spacing, so only the walked-record count can notice them
last = int(np.flatnonzero(g == g.max())[0])
t = 1 << 15
variants["hidden_block"] = np.concatenate([rec[:t + 50], rec[last:last + 100], rec[t + 50:last], rec[last + 100:]])
assert g[t - 1] == g[t + 60]
ctx = api.Context(0)
for name, r in variants.items():
    buf = torch.from_numpy(r.view(np.uint8).copy()).cuda()
    ctx.ingest([api.Segment(0, 0, 0, 128, 10, buf, len(r), flags=api.OWL_SEG_WARP_MAJOR)])
    try:
        ctx.build([0])
        print(name, "BUILT")
    except api.OwlError as e:
        print(name, str(e).split(":")[0])
    finally:
        ctx.forget_runs([0])
"""


def test_warp_major_misflag_detected():
    """Segments wrongly flagged OWL_SEG_WARP_MAJOR (> 2^15 records, several fold tiles) fail with
    OWL_ERR_INVALID_ARG: channel order, one warp's block moved inside another's, and a short block hidden just
    past a tile boundary.  No hang (the run is a subprocess under a timeout), no silently skipped record."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", _MISFLAG_SCRIPT.format(root=root)], capture_output=True, text=True,
                       timeout=300, cwd=root)
    assert r.returncode == 0, r.stderr
    lines = dict(ln.split(" ", 1) for ln in r.stdout.strip().splitlines())
    assert lines == {"interleaved": "OWL_ERR_INVALID_ARG", "split_warp": "OWL_ERR_INVALID_ARG",
                     "hidden_block": "OWL_ERR_INVALID_ARG"}, r.stdout


def test_channel_order_first_bad_record(ctx):
    """Channel order with two malformed records: the report names the first in the caller's order (as the oracle
    does), although bucketing by warp puts the other one first."""
    rec = tracegen.interleave(H.w1_records(), burst=2)
    w0 = [i for i in range(len(rec)) if rec["gwarp"][i] == 0 and rec["meta"][i] >> 31]
    w1 = [i for i in range(len(rec)) if rec["gwarp"][i] == 1 and rec["meta"][i] >> 31]
    late0, early1 = w0[-1], w1[0]
    assert early1 < late0
    for i in (late0, early1):
        rec["addr"][i] = np.uint64(12) << np.uint64(60)
    with pytest.raises(oracle.OracleError) as eo:
        oracle.build([oracle.Segment(0, 0, 0, 2, 10, rec)])
    assert f"record {early1}:" in str(eo.value)
    buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
    for mode in (api.OWL_CHANNEL_COPY, api.OWL_CHANNEL_IN_PLACE):
        ctx.set_config(channel_order=mode)
        ctx.ingest([api.Segment(0, 0, 0, 2, 10, buf, len(rec), flags=0)])
        try:
            with pytest.raises(api.OwlError, match="OWL_ERR_MALFORMED_TRACE") as eg:
                ctx.build([0])
            assert str(eo.value).split(": ", 1)[1] in str(eg.value)
        finally:
            ctx.forget_runs([0])
            ctx.set_config()


def test_host_records_channel_order_malformed_first_wave(ctx):
    """Host records in channel order staged in several waves, a malformed record in the first wave: the report
    (made after the last wave, through the bucketed records) names the oracle's record, although the first wave's
    staging buffer has been refilled by then."""
    ctx.set_config(host_chunk_bytes=1 << 20)
    p = tracegen.Params.preset(2, grid_div=64, runs_fix=4, runs_rnd=0)
    runs = list(range(p.n_runs))
    segs, osegs = [], []
    for r in runs:
        for m in tracegen.run_segments(p, r):
            rec = tracegen.interleave(tracegen.host_records(p, r, m.seq))
            if r == 0:
                i = int(np.flatnonzero(rec["meta"] >> 31)[5000])  # a MEM record
                rec["addr"][i] = np.uint64(12) << np.uint64(60)
            osegs.append(oracle.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, rec))
            host = torch.from_numpy(rec.view(np.uint8).copy()).pin_memory()
            segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, host, len(rec),
                                    flags=api.OWL_SEG_HOST_RECORDS))
    with pytest.raises(oracle.OracleError) as eo:
        oracle.build(osegs)
    ctx.ingest(segs)
    try:
        with pytest.raises(api.OwlError, match="OWL_ERR_MALFORMED_TRACE") as eg:
            ctx.build(runs)
        assert str(eo.value).split(": ", 1)[1] in str(eg.value), (str(eo.value), str(eg.value))
    finally:
        ctx.forget_runs(runs)
        ctx.set_config()


@pytest.mark.parametrize("cfg,div,interleaved,chunk", [(2, 32, False, 0), (5, 32, True, 0), (4, 256, False, 0),
                                                       (2, 32, False, 1 << 20), (5, 32, True, 1 << 20),
                                                       (9, 16, False, 3 << 20)])
def test_host_records_e2e_path(ctx, cfg, div, interleaved, chunk):
    """OWL_SEG_HOST_RECORDS (the bench's e2e leg): host buffers staged by the library give the oracle's result,
    in one wave or (small host_chunk_bytes) in many waves through the two staging buffers."""
    ctx.set_config(host_chunk_bytes=chunk)
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=2, runs_rnd=2)
    runs = list(range(p.n_runs))
    segs = []
    for r in runs:
        for m in tracegen.run_segments(p, r):
            rec = tracegen.host_records(p, r, m.seq)
            if interleaved:
                rec = tracegen.interleave(rec)
            host = torch.from_numpy(rec.view(np.uint8).copy()).pin_memory()
            flags = api.OWL_SEG_HOST_RECORDS | (0 if interleaved else api.OWL_SEG_WARP_MAJOR)
            segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, host, len(rec), flags=flags))
    ctx.ingest(segs)
    ctx.reset_stats()
    try:
        ef, er = ctx.build(_runs_of(p, 0)), ctx.build(_runs_of(p, 1))
        osg = _oracle_segments(p, runs)
        of, orr = oracle.build(osg[0]), oracle.build(osg[1])
        assert ef.export() == of.export() and er.export() == orr.export()
        assert_leak_parity(ctx.leak_test(ef, er, SIG), oracle.leak_test(of, orr, SIG))
        if chunk:
            assert ctx.stats()["fold_launches"] > 2  # several waves
    finally:
        ctx.forget_runs(runs)
        ctx.set_config()
