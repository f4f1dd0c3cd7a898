"""Test helpers: record construction, the canonical-dump parser, an independent pure-Python
per-warp walk (brute force for tiny traces) and random tiny trace generation."""
from __future__ import annotations

import json
import os
import struct
from collections import defaultdict

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
RECORD_DTYPE = np.dtype([("addr", "<u8"), ("gwarp", "<u4"), ("meta", "<u4")])
S = 0xFFFFFFFF


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def bb_rec(gwarp, bb):
    return (0, gwarp, (bb & 0x3FFFF) << 8)


def mem_rec(gwarp, bb, ins, lane, addr):
    return (addr, gwarp, 0x80000000 | ((lane & 31) << 26) | ((bb & 0x3FFFF) << 8) | (ins & 0xFF))


def to_records(rows):
    return np.array(rows, dtype=RECORD_DTYPE)


def w1_records(doc=None):
    doc = doc or load_golden("w1.json")
    rows = []
    for r in doc["records"]:
        if r[0] == "B":
            rows.append(bb_rec(r[1], r[2]))
        else:
            rows.append(mem_rec(r[1], r[2], r[3], r[4], r[5]))
    return to_records(rows)


# ---- canonical dump parser (format spec) ---------------------------------------------
SLOT_DT = np.dtype([("slot", "<u4"), ("_pad", "<u4"), ("kernel_id", "<u8"), ("count", "<u8")])
NODE_DT = np.dtype([("slot", "<u4"), ("bb", "<u4"), ("count", "<u8")])
EDGE_DT = np.dtype([("slot", "<u4"), ("src", "<u4"), ("dst", "<u4"), ("_pad", "<u4"), ("count", "<u8")])
TRIPLE_DT = np.dtype([("slot", "<u4"), ("bb", "<u4"), ("prev", "<u4"), ("next", "<u4"), ("count", "<u8")])
ADDR_DT = np.dtype([("slot", "<u4"), ("bb", "<u4"), ("ins", "<u4"), ("j", "<u4"), ("x", "<u8"), ("count", "<u8")])


def parse_blob(blob: bytes):
    assert blob[:8] == b"OWLADCFG", blob[:8]
    ver, cls, n_runs, n_slots = struct.unpack_from("<4I", blob, 8)
    n_node, n_edge, n_triple, n_addr = struct.unpack_from("<4Q", blob, 24)
    off = 56
    out = dict(version=ver, input_class=cls, n_runs=n_runs)
    for name, dt, n in (("slots", SLOT_DT, n_slots), ("node", NODE_DT, n_node), ("edge", EDGE_DT, n_edge),
                        ("triple", TRIPLE_DT, n_triple), ("addr", ADDR_DT, n_addr)):
        out[name] = np.frombuffer(blob, dtype=dt, count=n, offset=off)
        off += n * dt.itemsize
    assert off == len(blob)
    return out


def blob_tables_as_lists(p):
    return {
        "node": [[int(r["slot"]), int(r["bb"]), int(r["count"])] for r in p["node"]],
        "edge": [[int(r["slot"]), int(r["src"]), int(r["dst"]), int(r["count"])] for r in p["edge"]],
        "triple": [[int(r["slot"]), int(r["bb"]), int(r["prev"]), int(r["next"]), int(r["count"])] for r in p["triple"]],
        "addr": [[int(r["slot"]), int(r["bb"]), int(r["ins"]), int(r["j"]), int(r["x"]), int(r["count"])] for r in p["addr"]],
    }


# ---- independent brute-force per-warp walk, pure Python, tiny inputs only ----------------
def py_walk(records, slot=0):
    """Returns dict of Counter-like dicts keyed as the canonical tables."""
    node, edge, triple, addr = defaultdict(int), defaultdict(int), defaultdict(int), defaultdict(int)
    per_warp = defaultdict(list)
    for rec in records:
        per_warp[int(rec["gwarp"])].append(rec)
    for w, recs in per_warp.items():
        trace = []  # list of [bb, {(ins, x): count}]  — the warp trace T_w = (T_b1, T_b2, ...)
        for rec in recs:
            meta = int(rec["meta"])
            if meta >> 31 == 0:
                trace.append([(meta >> 8) & 0x3FFFF, defaultdict(int)])
            else:
                assert trace and trace[-1][0] == (meta >> 8) & 0x3FFFF
                trace[-1][1][(meta & 0xFF, int(rec["addr"]))] += 1
        seen = defaultdict(int)
        bbs = [t[0] for t in trace]
        for i, (b, mem) in enumerate(trace):
            seen[b] += 1
            node[(slot, b)] += 1
            src = bbs[i - 1] if i > 0 else S
            dst = bbs[i + 1] if i + 1 < len(bbs) else S
            edge[(slot, src, b)] += 1
            triple[(slot, b, src, dst)] += 1
            for (ins, x), c in mem.items():
                addr[(slot, b, ins, seen[b], x)] += c
        if bbs:
            edge[(slot, bbs[-1], S)] += 1
    return {
        "node": sorted([list(k) + [v] for k, v in node.items()]),
        "edge": sorted([list(k) + [v] for k, v in edge.items()]),
        "triple": sorted([list(k) + [v] for k, v in triple.items()]),
        "addr": sorted([list(k) + [v] for k, v in addr.items()]),
    }


def random_trace(rng: np.random.Generator, n_warps=4, max_bbs=6, n_bb_ids=5, max_ins=3, n_addr=6, active=0.7):
    """Random valid warp-major trace: each warp visits a random BB sequence; at each visit each
    instruction is executed by a random active subset of lanes, with addresses from a small pool."""
    rows = []
    for w in range(n_warps):
        nb = int(rng.integers(0, max_bbs + 1))
        for _ in range(nb):
            b = int(rng.integers(0, n_bb_ids))
            rows.append(bb_rec(w, b))
            for ins in range(int(rng.integers(0, max_ins + 1))):
                for lane in range(32):
                    if rng.random() < active:
                        x = int(rng.integers(0, n_addr)) * 4 | (3 << 60)
                        rows.append(mem_rec(w, b, ins, lane, x))
    return to_records(rows) if rows else np.zeros(0, dtype=RECORD_DTYPE)


def interleave_random(rng, rec):
    """A random interleaving of the warps' record streams that keeps each warp's order."""
    if len(rec) == 0:
        return rec.copy()
    by_w = defaultdict(list)
    for i, g in enumerate(rec["gwarp"]):
        by_w[int(g)].append(i)
    queues = [list(v) for v in by_w.values()]
    order = []
    while queues:
        k = int(rng.integers(0, len(queues)))
        order.append(queues[k].pop(0))
        if not queues[k]:
            queues.pop(k)
    return rec[np.array(order)]


# ---- hand-worked leak-test cases (tests/golden/leak_localization.json) ------------------------------
NA = 0xFFFFFFFF


def dsl_records(visits, n_warps):
    """Warp-major records of one invocation: every warp runs `visits` = [[bb, [[ins, lanes, base], ...]], ...];
    lane l < lanes of instruction ins accesses x = (3 << 60) | (base + 4 l)."""
    rows = []
    for w in range(n_warps):
        for bb, mems in visits:
            rows.append(bb_rec(w, bb))
            for ins, lanes, base in mems:
                for lane in range(lanes):
                    rows.append(mem_rec(w, bb, ins, lane, (3 << 60) | (base + 4 * lane)))
    return to_records(rows)


def golden_case_invocations(case):
    """[(run, class, seq, n_warps, kernel_id, records)] of a leak_localization.json case."""
    out = []
    for run, cls, names in case["runs"]:
        for seq, name in enumerate(names):
            nw = case["n_warps"][name]
            out.append((run, cls, seq, nw, case["kernels"][name], dsl_records(case["bodies"][name][str(cls)], nw)))
    return out


def golden_expected_rows(case):
    """Expected leak rows with NA / nan / closed-form p resolved: list of dicts."""
    import math
    rows = []
    for e in case["expected"]:
        r = {}
        for k, v in e.items():
            if k == "kernel":
                r["kernel_id"] = case["kernels"][v]
            elif v == "NA":
                r[k] = NA
            elif v == "nan":
                r[k] = float("nan")
            elif k == "p" and isinstance(v, str):
                assert v.startswith("2*exp(-") and v.endswith(")"), v
                r[k] = 2.0 * math.exp(-float(v[7:-1]))
            else:
                r[k] = v
        rows.append(r)
    return rows


def assert_leaks_equal_golden(got, case):
    """Every field of every leak row against the hand-worked expectation (p: closed form, 1e-12 relative)."""
    import math
    want = golden_expected_rows(case)
    assert len(got) == len(want), (len(got), len(want))
    for g, w in zip(got, want):
        for f in ("kind", "slot_fix", "slot_rnd", "bb", "ins", "j", "kernel_id", "n", "m"):
            assert int(g[f]) == int(w[f]), (f, int(g[f]), w)
        K = int(g["K_lo"]) | (int(g["K_hi"]) << 64)
        assert K == int(w["K"]), (K, w)
        for f in ("D", "p"):
            if math.isnan(w[f]):
                assert math.isnan(float(g[f])), (f, g[f], w)
            else:
                assert abs(float(g[f]) - w[f]) <= 1e-12 * abs(w[f]), (f, float(g[f]), w)
