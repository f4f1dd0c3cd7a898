"""H_cf reading R2: KS over the row-normalized control-flow transition matrix A.  TEST INFRASTRUCTURE ONLY.

May be imported only by tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
(same rule as oracle.py).  Pure Python with exact rationals (fractions.Fraction); shares nothing with the
CUDA path.  SURVEY §8(f) N3, reading R22.

Paper, P:L280-296 (§VII.B, Eqs. 5-8):
  * node N executed n times, each execution a (src, dst) pair; I = (x_1..x_k) the src counts, sum x_i = n
    (Eq. 5); O = (y_1..y_p) the dst counts (Eq. 6);
  * A (k x p) with I . A = O (Eq. 7), "a feasible solution by counting the number of each type of
    (src, dst)": a_ij = c_ij / x_i, c_ij the joint count (then sum_i x_i a_ij = sum_i c_ij = y_j);
  * H = (a_11, a_12, ..., a_1p, a_21, ..., a_kp) (Eq. 8): x-axis the control flow (src, dst) in row-major
    order (S last, reading R6), y-axis the element of A.
KS (Eqs. 1-4) of the fix and rnd histograms, each a weighted sample with weights a_ij:
  F(t) = sum_{cells <= t} a_ij / sum_all a_ij,  D = max over the union of cells of |F_fix - F_rnd|,
  sample sizes n, m = the node counts (Eq. 5; reading R22), p = 2 exp(-2 D^2 n m / (n + m)) (Eq. 4),
  fail iff p < significance (reading R1).
D is computed exactly as a rational and rounded once to fp64; p follows Eq. 4 in fp64 in the order of
DESIGN.md §3.
"""
from __future__ import annotations

import math
from fractions import Fraction


def transition_matrix(cells):
    """cells: [(src, dst, c_ij)] of one node.  Returns {(src, dst): a_ij} with a_ij = c_ij / x_i (Eq. 7)."""
    x = {}
    for s, _, c in cells:
        x[s] = x.get(s, 0) + c  # Eq. 5: x_i = count of src i
    return {(s, d): Fraction(c, x[s]) for s, d, c in cells}


def ks_r2(cells_fix, cells_rnd, significance: float = 0.05):
    """One H_cf test under R2.  Returns (n, m, D_exact, D, p, fail)."""
    a_f, a_r = transition_matrix(cells_fix), transition_matrix(cells_rnd)
    n = sum(c for _, _, c in cells_fix)
    m = sum(c for _, _, c in cells_rnd)
    tot_f, tot_r = sum(a_f.values()), sum(a_r.values())
    D = Fraction(0)
    for t in sorted(set(a_f) | set(a_r)):  # (src, dst) row-major; S = 0xFFFFFFFF sorts last
        F_f = sum((a for key, a in a_f.items() if key <= t), Fraction(0)) / tot_f
        F_r = sum((a for key, a in a_r.items() if key <= t), Fraction(0)) / tot_r
        D = max(D, abs(F_f - F_r))
    Dd = float(D)
    nd, md = float(n), float(m)
    nm = nd * md
    w = nm / (nd + md)
    x = (2.0 * (Dd * Dd)) * w
    p = 2.0 * math.exp(-x)
    return n, m, D, Dd, p, p < significance


def node_cells(triples, slot, bb):
    """The (prev, next, count) cells of node (slot, bb) from a parsed canonical triple table."""
    sel = (triples["slot"] == slot) & (triples["bb"] == bb)
    t = triples[sel]
    return [(int(r["prev"]), int(r["next"]), int(r["count"])) for r in t]
