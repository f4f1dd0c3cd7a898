"""The O6 / O8 pins have teeth: deliberately broken builds of the oracle (one plausible mistake each in the
kernel leak test, P:L278 / R12, or the leak localization, P:L299-301 / R14) must FAIL the hand-worked
cases of tests/golden/leak_localization.json.  Each mutant is a textual edit of oracle/owl_oracle.cpp
compiled into a temporary library; the committed oracle itself is never changed."""
import ctypes
import gc
import os
import subprocess

import pytest

from oracle import oracle
from tests import helpers as H

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "owl_oracle.cpp")
DOC = H.load_golden("leak_localization.json")

MUTANTS = {
    # O6: raw invocation counts instead of count_f * R_rnd vs count_r * R_fix (reading R12)
    "raw_counts": ("(u128)f.slot_count[sf] * r.n_runs != (u128)r.slot_count[sr] * f.n_runs",
                   "f.slot_count[sf] != r.slot_count[sr]"),
    # O6: n / m of an unaligned evidence slot swapped
    "del_counts_swapped": ("f.slot_kid[s], f.slot_count[s], 0ull,", "f.slot_kid[s], 0ull, f.slot_count[s],"),
    # O6: slot fields of an unaligned run invocation swapped
    "ins_slots_swapped": ("kern.push_back({0u, NA, s,", "kern.push_back({0u, s, NA,"),
    # O8: the max-p visit represents the location
    "max_p": ("k.p < rows[it->second].p", "k.p > rows[it->second].p"),
    # O8: the first failing visit represents the location
    "first_fail": ("if (it == df_best.end() || k.p < rows[it->second].p)", "if (it == df_best.end())"),
    # O8: ties go to the largest j
    "ties_largest_j": ("k.p < rows[it->second].p", "k.p <= rows[it->second].p"),
    # O8: DF rows ordered by fix slot id instead of alignment position
    "order_by_slot": ("auto key = std::make_tuple(pos[i], k.bb, k.ins);",
                      "auto key = std::make_tuple((int)k.slot_fix, k.bb, k.ins);"),
}


def _build_mutant(tmp_path, name):
    old, new = MUTANTS[name]
    src = open(SRC).read()
    assert src.count(old) == 1, f"mutation site of {name} not found exactly once"
    path = tmp_path / f"owl_oracle_{name}.cpp"
    path.write_text(src.replace(old, new))
    so = tmp_path / f"liboracle_{name}.so"
    subprocess.run(["g++", "-std=c++17", "-O1", "-ffp-contract=off", "-fPIC", "-shared", "-pthread", "-o", str(so),
                    str(path)], check=True)
    return oracle.bind(ctypes.CDLL(str(so)))


def _case_passes(case):
    by_cls = {0: [], 1: []}
    for run, cls, seq, nw, kid, rec in H.golden_case_invocations(case):
        by_cls[cls].append(oracle.Segment(run, cls, seq, nw, kid, rec))
    f, r = oracle.build(by_cls[0]), oracle.build(by_cls[1])
    got = oracle.leak_test(f, r, 0.05)
    del f, r
    gc.collect()
    try:
        H.assert_leaks_equal_golden(got, case)
        return True
    except AssertionError:
        return False


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_mutant_fails_a_pin(tmp_path, monkeypatch, name):
    mutant = _build_mutant(tmp_path, name)
    monkeypatch.setattr(oracle, "_lib", mutant)
    try:
        results = {c: _case_passes(DOC["cases"][c]) for c in sorted(DOC["cases"])}
    finally:
        gc.collect()
    assert not all(results.values()), f"mutant {name} passes every hand-worked case: {results}"


def test_unmutated_oracle_passes():
    assert all(_case_passes(DOC["cases"][c]) for c in sorted(DOC["cases"]))
