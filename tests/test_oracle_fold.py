"""Pins of the oracle's A-DCFG construction (O1-O5) against what the paper fixes (CPU only).

* W1: hand-worked tables (tests/golden/w1.json).
* Invariance under warp interleaving (warps are simultaneous), lane permutation (P:L185:
  predicated execution, one control flow per warp) and warp relabeling (warps are identified,
  not ordered).
* Conservation laws of Eqs. 5-6 (sum of src counts = n = sum of dst counts per node), plus
  record counts.
* An independent brute-force walk (tests/helpers.py::py_walk, an offline formulation over the list of
  BB visits) on random tiny traces.
* Evidence = sum of per-run A-DCFGs for aligned slots; identical inputs => zero differences
  (P:L229).
"""
import numpy as np
import pytest

import tracegen
from oracle import oracle
from tests import helpers as H


def _seg(rec, run=0, cls=0, seq=0, n_warps=2, kid=10):
    return oracle.Segment(run, cls, seq, n_warps, kid, rec)


def test_w1_hand_worked_tables():
    doc = H.load_golden("w1.json")
    rec = H.w1_records(doc)
    sg = doc["segment"]
    g = oracle.build([_seg(rec, sg["run"], sg["input_class"], sg["seq"], sg["n_warps"], sg["kernel_id"])])
    p = H.parse_blob(g.export())
    got = H.blob_tables_as_lists(p)
    for t in ("node", "edge", "triple", "addr"):
        assert got[t] == doc["expected"][t], t
    assert p["n_runs"] == 1 and len(p["slots"]) == 1
    assert int(p["slots"][0]["kernel_id"]) == 10 and int(p["slots"][0]["count"]) == 1


def test_w1_invariances():
    rec = H.w1_records()
    ref = oracle.build([_seg(rec)]).export()
    rng = np.random.default_rng(1)
    for _ in range(20):  # interleavings that keep each warp's order
        assert oracle.build([_seg(H.interleave_random(rng, rec))]).export() == ref
    swapped = rec.copy()  # lane swap 0 <-> 1
    m = swapped["meta"]
    is_mem = (m >> 31) == 1
    lane = (m >> 26) & 31
    newlane = np.where(lane == 0, 1, np.where(lane == 1, 0, lane))
    swapped["meta"] = np.where(is_mem, (m & ~np.uint32(31 << 26)) | (newlane.astype(np.uint32) << 26), m)
    assert oracle.build([_seg(swapped)]).export() == ref
    relabel = rec.copy()  # gwarp 0 <-> 1
    relabel["gwarp"] = 1 - relabel["gwarp"]
    assert oracle.build([_seg(relabel)]).export() == ref


def test_w1_malformed_variants():
    rec = H.w1_records()
    # a MEM record moved before its warp's first BB_ENTRY
    bad = np.concatenate([rec[1:2], rec[0:1], rec[2:]])
    with pytest.raises(oracle.OracleError, match="before the warp's first BB_ENTRY"):
        oracle.build([_seg(bad)])
    # a MEM record whose bb is not the warp's current BB
    bad = rec.copy()
    bad["meta"][4] = (bad["meta"][4] & ~np.uint32(0x3FFFF << 8)) | np.uint32(2 << 8)
    with pytest.raises(oracle.OracleError, match="bb != the warp's current BB"):
        oracle.build([_seg(bad)])
    bad = rec.copy()
    bad["gwarp"][3] = 7
    with pytest.raises(oracle.OracleError, match="gwarp >= n_warps"):
        oracle.build([_seg(bad)])
    bad = rec.copy()
    bad["addr"][0] = 5  # BB_ENTRY with a non-zero address
    with pytest.raises(oracle.OracleError, match="BB_ENTRY"):
        oracle.build([_seg(bad)])
    bad = rec.copy()
    bad["addr"][1] = np.uint64(9) << np.uint64(60)  # memory type 9 does not exist
    with pytest.raises(oracle.OracleError, match="memory type"):
        oracle.build([_seg(bad)])


def _conservation(rec, p, n_warps_with_bb):
    n_bb = int(np.sum((rec["meta"] >> 31) == 0))
    n_mem = len(rec) - n_bb
    node, edge, triple, addr = p["node"], p["edge"], p["triple"], p["addr"]
    assert int(node["count"].sum()) == n_bb
    assert int(edge["count"].sum()) == n_bb + n_warps_with_bb
    assert int(triple["count"].sum()) == n_bb
    assert int(addr["count"].sum()) == n_mem
    S = H.S
    assert int(edge["count"][edge["src"] == S].sum()) == n_warps_with_bb
    assert int(edge["count"][edge["dst"] == S].sum()) == n_warps_with_bb
    for r in node:  # Eqs. 5-6: sum_i x_i = n = sum_j y_j for each node
        s, b, c = int(r["slot"]), int(r["bb"]), int(r["count"])
        ins = int(edge["count"][(edge["slot"] == s) & (edge["dst"] == b)].sum())
        outs = int(edge["count"][(edge["slot"] == s) & (edge["src"] == b)].sum())
        tri = int(triple["count"][(triple["slot"] == s) & (triple["bb"] == b)].sum())
        assert ins == c == outs == tri


@pytest.mark.parametrize("seed", range(40))
def test_random_tiny_traces_brute_force(seed):
    rng = np.random.default_rng(seed)
    rec = H.random_trace(rng, n_warps=int(rng.integers(1, 6)))
    g = oracle.build([_seg(rec, n_warps=8)])
    p = H.parse_blob(g.export())
    assert H.blob_tables_as_lists(p) == H.py_walk(rec)
    n_w = len({int(w) for w in rec["gwarp"]})
    _conservation(rec, p, n_w)
    # interleaving invariance on random traces too
    assert oracle.build([_seg(H.interleave_random(rng, rec), n_warps=8)]).export() == g.export()


def test_generator_configs_conservation_and_brute_force():
    for cfg in (1, 2, 3, 4, 5):
        p = tracegen.Params.preset(cfg, grid_div=64 if cfg != 1 else 1, runs_fix=1, runs_rnd=1)
        for r in range(2):
            for m in tracegen.run_segments(p, r):
                rec = tracegen.host_records(p, r, m.seq)
                if len(rec) > 400_000:
                    rec = rec[rec["gwarp"] < 2]  # keep two whole warps
                g = oracle.build([oracle.Segment(r, m.input_class, 0, m.n_warps, m.kernel_id, rec)])
                pb = H.parse_blob(g.export())
                _conservation(rec, pb, len({int(w) for w in rec["gwarp"]}))
                if len(rec) < 60_000:
                    assert H.blob_tables_as_lists(pb) == H.py_walk(rec)


def _class_segments(p, cls, runs=None):
    out = []
    for r in (runs if runs is not None else range(p.n_runs)):
        for m in tracegen.run_segments(p, r):
            if m.input_class == cls:
                out.append(oracle.Segment(r, cls, m.seq, m.n_warps, m.kernel_id, tracegen.host_records(p, r, m.seq)))
    return out


def test_evidence_is_sum_of_runs_when_aligned():
    """aligned invocations' A-DCFGs are summed; counts are integers so the order is irrelevant."""
    p = tracegen.Params.preset(1)
    segs = _class_segments(p, 1)
    ev = H.parse_blob(oracle.build(segs).export())
    acc = {}
    for sg in segs:
        one = H.parse_blob(oracle.build([sg]).export())
        for t, key in (("node", ("slot", "bb")), ("edge", ("slot", "src", "dst")),
                       ("triple", ("slot", "bb", "prev", "next")), ("addr", ("slot", "bb", "ins", "j", "x"))):
            for row in one[t]:
                k = (t,) + tuple(int(row[f]) for f in key)
                acc[k] = acc.get(k, 0) + int(row["count"])
    got = {}
    for t, key in (("node", ("slot", "bb")), ("edge", ("slot", "src", "dst")),
                   ("triple", ("slot", "bb", "prev", "next")), ("addr", ("slot", "bb", "ins", "j", "x"))):
        for row in ev[t]:
            got[(t,) + tuple(int(row[f]) for f in key)] = int(row["count"])
    assert got == acc
    assert int(ev["slots"][0]["count"]) == len(segs) and ev["n_runs"] == len(segs)


def test_identical_inputs_zero_diff_and_mirror():
    p = tracegen.Params.preset(1)
    a = oracle.build(_class_segments(p, 1))
    b = oracle.build(_class_segments(p, 1))
    assert len(oracle.diff(a, b)) == 0 and a.export() == b.export()
    f = oracle.build(_class_segments(p, 0))
    d1, d2 = oracle.diff(f, a), oracle.diff(a, f)
    assert len(d1) > 0 and len(d1) == len(d2)
    assert np.array_equal(d1["count_a"], d2["count_b"]) and np.array_equal(d1["count_b"], d2["count_a"])
    # rows are exactly the symmetric difference of the two canonical dumps' cells
    pf, pa = H.parse_blob(f.export()), H.parse_blob(a.export())
    cells_f = {(t, tuple(r)) for t, rows in H.blob_tables_as_lists(pf).items() for r in rows}
    cells_a = {(t, tuple(r)) for t, rows in H.blob_tables_as_lists(pa).items() for r in rows}
    keys_changed = {(t, c[:-1]) for t, c in cells_f ^ cells_a}
    assert len([r for r in d1 if r["table"] != 4]) == len(keys_changed)


def test_fix_runs_are_identical_traces():
    """FIX runs of the deterministic configs repeat one secret: per-run A-DCFGs have no differences
    (the input-class filtering premise)."""
    p = tracegen.Params.preset(2, grid_div=128, runs_fix=2, runs_rnd=2)
    segs = _class_segments(p, 0)
    a, b = oracle.build([segs[0]]), oracle.build([oracle.Segment(0, 0, 0, segs[1].n_warps, segs[1].kernel_id, segs[1].records)])
    assert len(oracle.diff(a, b)) == 0
