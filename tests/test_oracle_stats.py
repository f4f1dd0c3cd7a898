"""Pins of the oracle's KS test (O7, Eqs. 1-4), Myers alignment (O4/O6) and the
whole-pipeline invariants (CPU only).

KS pins: the worked values (tests/golden/ks_examples.json), closed forms (D = 0 => p = 2; disjoint
supports => D = 1, p = 2 exp(-2nm/(n+m))), D equal to scipy.stats.ks_2samp on the expanded samples and to
the exact sup over all t computed with Fractions, and Eq. 3 <=> Eq. 4 at significance 0.05 (reading R1).
Myers pins: the worked examples M1-M3, script validity and shortest length (= N + M - 2 LCS by DP).
"""
import math
from fractions import Fraction

import numpy as np
import pytest
from scipy import stats

import tracegen
from oracle import oracle
from tests import helpers as H


def test_ks_worked_examples():
    doc = H.load_golden("ks_examples.json")
    for c in doc["cases"]:
        def enc(cells):
            xs = []
            for x, _ in cells:
                xs.append((x[0] << 32) | x[1] if isinstance(x, list) else x)  # (src,dst) row-major (R6)
            return xs, [n for _, n in cells]
        xf, cf = enc(c["fix"])
        xr, cr = enc(c["rnd"])
        row = oracle.ks_hist(xf, cf, xr, cr, 0.05)
        K = int(row["K_lo"]) | (int(row["K_hi"]) << 64)
        assert (int(row["n"]), int(row["m"]), K) == (c["n"], c["m"], c["K"]), c["id"]
        assert float(row["D"]) == c["D"], c["id"]
        assert float(row["p"]) == pytest.approx(c["p"], rel=1e-12), c["id"]
        assert bool(row["fail"]) == c["fail"], c["id"]
        # closed form of Eq. 4 from the printed D
        n, m = c["n"], c["m"]
        assert float(row["p"]) == pytest.approx(2 * math.exp(-2 * c["D"] ** 2 * n * m / (n + m)), rel=1e-12)


def test_ks_order_matters_example():
    """KS-3: the statistic depends on the category order, so the order must be fixed (R6)."""
    a, b, c = 1, 2, 3
    r1 = oracle.ks_hist([a, c], [1, 1], [b], [2])
    assert float(r1["D"]) == 0.5
    r2 = oracle.ks_hist([b, c], [1, 1], [a], [2])  # relabel so that the rnd category sorts first
    assert float(r2["D"]) == 1.0


def _expand(xs, cs):
    return np.repeat(np.asarray(xs, dtype=np.float64), np.asarray(cs, dtype=np.int64))


@pytest.mark.parametrize("seed", range(300))
def test_ks_statistic_brute_force(seed):
    rng = np.random.default_rng(seed)
    kf, kr = int(rng.integers(1, 7)), int(rng.integers(1, 7))
    pool = np.sort(rng.choice(20, size=12, replace=False))
    xf = np.sort(rng.choice(pool, size=kf, replace=False)); cf = rng.integers(1, 9, size=kf)
    xr = np.sort(rng.choice(pool, size=kr, replace=False)); cr = rng.integers(1, 9, size=kr)
    row = oracle.ks_hist(xf, cf, xr, cr, 0.05)
    n, m = int(cf.sum()), int(cr.sum())
    # exact sup over all t (Eqs. 1-2) with rationals
    ts = sorted(set(xf.tolist()) | set(xr.tolist()))
    Dx = max(abs(Fraction(int(cf[xf <= t].sum()), n) - Fraction(int(cr[xr <= t].sum()), m)) for t in ts)
    K = int(row["K_lo"])
    assert Fraction(K, n * m) == Dx
    assert float(row["D"]) == K / (float(n) * float(m))
    assert float(row["D"]) == pytest.approx(stats.ks_2samp(_expand(xf, cf), _expand(xr, cr)).statistic, abs=1e-15)
    # Eq. 3 <=> Eq. 4 at significance a = 0.05 (reading R1), away from the exact boundary
    a = 0.05
    thr = math.sqrt(-math.log(a / 2) * 0.5) * math.sqrt((n + m) / (n * m))
    if abs(float(row["D"]) - thr) > 1e-9:
        assert bool(row["fail"]) == (float(row["D"]) > thr)
    assert bool(row["fail"]) == (float(row["p"]) < a)


def test_ks_closed_forms():
    r = oracle.ks_hist([5, 9], [3, 4], [5, 9], [6, 8])  # same distribution => D = 0, p = 2 (R3)
    assert float(r["D"]) == 0.0 and float(r["p"]) == 2.0 and not r["fail"]
    for n, m in ((1, 1), (7, 3), (100, 100), (1000, 10)):
        r = oracle.ks_hist([1], [n], [2], [m])
        assert float(r["D"]) == 1.0
        assert float(r["p"]) == pytest.approx(2 * math.exp(-2 * n * m / (n + m)), rel=1e-13)
    # 128-bit K: counts near 2^40 on both sides
    big = 1 << 40
    r = oracle.ks_hist([1, 2], [big, 1], [1, 2], [1, big])
    K = int(r["K_lo"]) | (int(r["K_hi"]) << 64)
    n = m = big + 1
    assert K == abs(big * m - 1 * n)


def test_myers_worked_examples():
    doc = H.load_golden("myers_examples.json")
    for c in doc["cases"]:
        enc = {k: i + 1 for i, k in enumerate("ABCD")}
        ops = oracle.myers([enc[k] for k in c["evidence"]], [enc[k] for k in c["run"]])
        assert [list(o) for o in ops] == c["script"], c["id"]


def _lcs(a, b):
    L = [[0] * (len(b) + 1) for _ in range(len(a) + 1)]
    for i in range(len(a)):
        for j in range(len(b)):
            L[i + 1][j + 1] = L[i][j] + 1 if a[i] == b[j] else max(L[i][j + 1], L[i + 1][j])
    return L[-1][-1]


@pytest.mark.parametrize("seed", range(200))
def test_myers_valid_and_shortest(seed):
    rng = np.random.default_rng(seed)
    a = rng.integers(0, 3, size=int(rng.integers(0, 9))).tolist()
    b = rng.integers(0, 3, size=int(rng.integers(0, 9))).tolist()
    ops = oracle.myers(a, b)
    i = j = 0
    nd = 0
    seen_ins_in_stretch = False
    for t, oi, oj in ops:
        if t == "M":
            assert (oi, oj) == (i, j) and a[i] == b[j]
            i += 1; j += 1
            seen_ins_in_stretch = False
        elif t == "D":
            assert oi == i and not seen_ins_in_stretch  # deletions precede insertions (R11)
            i += 1; nd += 1
        else:
            assert oj == j
            j += 1; nd += 1
            seen_ins_in_stretch = True
    assert (i, j) == (len(a), len(b))
    assert nd == len(a) + len(b) - 2 * _lcs(a, b)


def _mk_run(run, cls, kids):
    segs = []
    for s, k in enumerate(kids):
        rec = H.to_records([H.bb_rec(0, 1), H.mem_rec(0, 1, 0, 0, 0x40 + k)])
        segs.append(oracle.Segment(run, cls, s, 1, k, rec))
    return segs


def test_evidence_merge_examples():
    """M1-M3 through the evidence merge: slot order, new-slot ids, counts."""
    doc = H.load_golden("myers_examples.json")
    enc = {k: i + 1 for i, k in enumerate("ABCD")}
    for c in doc["cases"]:
        segs = _mk_run(0, 0, [enc[k] for k in c["evidence"]]) + _mk_run(1, 0, [enc[k] for k in c["run"]])
        ev = oracle.build(segs)
        slots, kids, counts = ev.slots()
        assert [int(k) for k in kids] == [enc[k] for k in c["order_kernels"]], c["id"]
        if "slot_counts" in c:
            assert [int(x) for x in counts] == c["slot_counts"]
        else:
            assert {k: int(counts[list(kids).index(enc[k])]) for k in c["counts"]} == c["counts"]
        # new slots get ids in creation order after the first run's slots
        assert sorted(int(s) for s in slots) == list(range(len(slots)))


def _class_segs(p, cls):
    out = []
    for r in range(p.n_runs):
        for m in tracegen.run_segments(p, r):
            if m.input_class == cls:
                out.append(oracle.Segment(r, cls, m.seq, m.n_warps, m.kernel_id, tracegen.host_records(p, r, m.seq)))
    return out


def test_identical_classes_no_leaks():
    """North-star invariant: identical inputs => zero differences and no leaks; every D = 0."""
    p = tracegen.Params.preset(1)
    a, b = oracle.build(_class_segs(p, 0)), oracle.build(_class_segs(p, 0))
    ks = oracle.ks_tests(a, b)
    assert len(ks) > 0 and np.all(ks["D"] == 0.0) and np.all(ks["p"] == 2.0)
    assert len(oracle.leak_test(a, b)) == 0


def test_planted_leaks_c1():
    """Sanity against the generator's ground truth (not parity): C1 plants a CF leak at B0 and DF leaks
    at the T-table instructions of B1/B3."""
    p = tracegen.Params.preset(1)
    f, r = oracle.build(_class_segs(p, 0)), oracle.build(_class_segs(p, 1))
    lk = oracle.leak_test(f, r)
    cf = {(int(x["bb"])) for x in lk if x["kind"] == 1}
    df = {(int(x["bb"]), int(x["ins"])) for x in lk if x["kind"] == 2}
    assert 0 in cf
    # 10 + 10 runs of 256 threads: most (not necessarily all) T-table instructions fail at a = 0.05
    assert sum((3, i) in df for i in range(8)) >= 5 and sum((1, i) in df for i in range(8)) >= 4
    assert not any(x["kind"] == 0 for x in lk)
    ks = oracle.ks_tests(f, r)
    det = ks[(ks["kind"] == 2) & (((ks["bb"] == 0)) | ((ks["bb"] == 3) & (ks["ins"] == 9)))]
    assert len(det) == 3 and np.all(det["D"] == 0.0)  # deterministic accesses: D = 0


def test_planted_kernel_leak_c4():
    p = tracegen.Params.preset(4, grid_div=256, runs_fix=4, runs_rnd=4)
    f, r = oracle.build(_class_segs(p, 0)), oracle.build(_class_segs(p, 1))
    lk = oracle.leak_test(f, r)
    kern = [x for x in lk if x["kind"] == 0]
    n_zero = sum(tracegen.run_segments(p, rr)[-1].seq < 3 for rr in range(p.n_runs) if tracegen.run_class(p, rr) == 1)
    assert (len(kern) > 0) == (n_zero > 0)
