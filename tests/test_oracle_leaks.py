"""Pins of the oracle's kernel leak test (O6, reading R12) and leak localization (O8, P:L299, P:L301,
reading R14) against hand-worked cases (tests/golden/leak_localization.json): every field of every row.

A plausible mistake fails one of them: comparing raw invocation counts instead of count_f*R_rnd vs
count_r*R_fix (K1 slots A and B), wrong slot / count fields of unaligned rows (K1 D and C), the first failing
visit or the max-p visit instead of the min-p one (L1 bb1 ins0), ties to the largest j (L1 bb1 ins1), only
j = 1 considered (L1 bb1 ins2), rows ordered by slot id instead of alignment position (L1: B's fix slot 1
precedes A's fix slot 0)."""
import pytest

from oracle import oracle
from tests import helpers as H

DOC = H.load_golden("leak_localization.json")


def _oracle_leaks(case):
    by_cls = {0: [], 1: []}
    for run, cls, seq, nw, kid, rec in H.golden_case_invocations(case):
        by_cls[cls].append(oracle.Segment(run, cls, seq, nw, kid, rec))
    f, r = oracle.build(by_cls[0]), oracle.build(by_cls[1])
    return oracle.leak_test(f, r, 0.05), f, r


@pytest.mark.parametrize("name", sorted(DOC["cases"]))
def test_oracle_leak_rows_match_hand_worked(name):
    case = DOC["cases"][name]
    got, _, _ = _oracle_leaks(case)
    H.assert_leaks_equal_golden(got, case)


def test_l1_slot_order_differs_from_alignment_order():
    """The case is only a pin of the row order if slot ids and alignment positions disagree."""
    _, f, r = _oracle_leaks(DOC["cases"]["L1"])
    slots, kids, _ = f.slots()
    assert list(slots) == [1, 0] and list(kids) == [11, 10]


def test_k1_counts_and_run_numbers():
    _, f, r = _oracle_leaks(DOC["cases"]["K1"])
    assert list(f.slots()[2]) == [2, 2, 2] and list(r.slots()[2]) == [3, 2, 2]
    assert list(r.slots()[1]) == [10, 11, 12]
