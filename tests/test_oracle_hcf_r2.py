"""Pins of the R2 H_cf oracle (oracle/hcf_r2.py, Eqs. 5-8), CPU only.

* hand-worked values (tests/golden/hcf_r2_examples.json);
* I . A = O (Eq. 7) for the constructed A, and every row of A sums to 1;
* a node with one src reduces to the plain count KS (R1), checked against the C++ oracle's ks_hist, whose own
  pins are in test_oracle_stats.py;
* brute force: each cell replicated L * a_ij times (L = the lcm of the row totals, an integer weight) is an
  ordinary sample whose two-sample KS D (scipy.stats.ks_2samp) equals the R2 D;
* scaling a row of counts leaves D unchanged (only A enters), while R1's D changes.
"""
import math
import random
from fractions import Fraction

import numpy as np
import pytest
from scipy import stats

from oracle import hcf_r2, oracle
from tests import helpers as H


def test_worked_examples():
    doc = H.load_golden("hcf_r2_examples.json")
    for c in doc["cases"]:
        fix = [tuple(x) for x in c["fix"]]
        rnd = [tuple(x) for x in c["rnd"]]
        n, m, D, Dd, p, fail = hcf_r2.ks_r2(fix, rnd)
        assert (n, m) == (c["n"], c["m"]), c["name"]
        assert D == Fraction(c["D"]), c["name"]
        assert Dd == float(Fraction(c["D"]))


def _random_node(rng, srcs=4, dsts=4, maxc=9):
    cells = set()
    for _ in range(rng.randint(1, srcs * dsts)):
        cells.add((rng.choice([1, 2, 3, 7, 0xFFFFFFFF][:srcs + 1]), rng.choice([2, 3, 5, 0xFFFFFFFF][:dsts])))
    return sorted((s, d, rng.randint(1, maxc)) for s, d in cells)


def test_transition_matrix_eq7():
    rng = random.Random(7)
    for _ in range(50):
        cells = _random_node(rng)
        A = hcf_r2.transition_matrix(cells)
        x, y = {}, {}
        for s, d, c in cells:
            x[s] = x.get(s, 0) + c
            y[d] = y.get(d, 0) + c
        for s in x:  # rows of A sum to 1
            assert sum(a for (si, _), a in A.items() if si == s) == 1
        for d in y:  # I . A = O
            assert sum(x[s] * a for (s, dj), a in A.items() if dj == d) == y[d]


def test_single_src_equals_count_ks():
    rng = random.Random(11)
    for _ in range(40):
        f = [(3, d, c) for _, d, c in _random_node(rng, srcs=1)]
        f = sorted({(s, d): c for s, d, c in f}.items())
        f = [(s, d, c) for (s, d), c in f]
        r = [(3, d, rng.randint(1, 9)) for d in sorted({rng.choice([2, 5, 9, 0xFFFFFFFF]) for _ in range(3)})]
        n, m, D, Dd, p, fail = hcf_r2.ks_r2(f, r)
        o = oracle.ks_hist([(s << 32) | d for s, d, _ in f], [c for *_, c in f],
                           [(s << 32) | d for s, d, _ in r], [c for *_, c in r])
        assert int(o["n"]) == n and int(o["m"]) == m
        assert float(o["D"]) == Dd
        assert float(o["p"]) == p


def test_brute_force_replicated_samples():
    rng = random.Random(3)
    for _ in range(60):
        f, r = _random_node(rng), _random_node(rng)
        _, _, D, Dd, _, _ = hcf_r2.ks_r2(f, r)

        rank = {k: i for i, k in enumerate(sorted({(s, d) for s, d, _ in f + r}))}  # exact in float64

        def sample(cells):
            A = hcf_r2.transition_matrix(cells)
            L = math.lcm(*[a.denominator for a in A.values()])
            out = []
            for key, a in sorted(A.items()):
                out += [rank[key]] * int(a * L)
            return np.array(out, dtype=np.float64)

        res = stats.ks_2samp(sample(f), sample(r), method="asymp")
        assert abs(res.statistic - float(D)) <= 1e-12, (f, r, D, res.statistic)


def test_row_scaling_invariance():
    rng = random.Random(5)
    for _ in range(30):
        f = _random_node(rng)
        s0 = f[0][0]
        g = [(s, d, c * 7 if s == s0 else c) for s, d, c in f]
        assert hcf_r2.ks_r2(f, g)[2] == 0
    # R1 sees the scaling when another row exists
    f = [(1, 2, 1), (1, 3, 1), (2, 3, 4)]
    g = [(1, 2, 7), (1, 3, 7), (2, 3, 4)]
    o = oracle.ks_hist([(s << 32) | d for s, d, _ in f], [c for *_, c in f],
                       [(s << 32) | d for s, d, _ in g], [c for *_, c in g])
    assert float(o["D"]) > 0 and hcf_r2.ks_r2(f, g)[2] == 0
