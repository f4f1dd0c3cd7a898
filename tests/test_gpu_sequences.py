"""GPU parity of the evidence merge and the leak test on realistic kernel sequences (Myers; kernel
leaks; localization): repeated kernel ids, mid-sequence insertions and deletions, slot ids
that differ from alignment positions.  Through the C ABI, against the oracle and the hand-worked cases."""
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
from tests.gpu_common import SIG, _build_and_compare, assert_ks_parity, assert_leak_parity  # noqa: E402

DOC = H.load_golden("leak_localization.json")


@pytest.fixture(scope="module")
def ctx():
    return api.Context(0)


def _ingest_invocations(ctx, invs):
    segs = []
    for run, cls, seq, nw, kid, rec in invs:
        buf = torch.from_numpy(rec.view(np.uint8).copy()).cuda()
        segs.append(api.Segment(run, cls, seq, nw, kid, buf, len(rec)))
    ctx.ingest(segs)
    return segs


def _compare_invocations(ctx, invs):
    """E_fix / E_rnd of the given invocations: GPU = oracle (dumps, KS rows, leaks, diff)."""
    _ingest_invocations(ctx, invs)
    runs = sorted({i[0] for i in invs})
    try:
        rf = sorted({i[0] for i in invs if i[1] == 0})
        rr = sorted({i[0] for i in invs if i[1] == 1})
        ef, er = ctx.build(rf), ctx.build(rr)
        osg = {0: [], 1: []}
        for run, cls, seq, nw, kid, rec in invs:
            osg[cls].append(oracle.Segment(run, cls, seq, nw, kid, rec))
        of, orr = oracle.build(osg[0]), oracle.build(osg[1])
        assert ef.export() == of.export()
        assert er.export() == orr.export()
        assert_ks_parity(ctx.ks_tests(ef, er, SIG), oracle.ks_tests(of, orr, SIG))
        gl = ctx.leak_test(ef, er, SIG)
        assert_leak_parity(gl, oracle.leak_test(of, orr, SIG))
        gd, od = ctx.diff(ef, er), oracle.diff(of, orr)
        assert len(gd) == len(od) and np.array_equal(gd, od)
        return gl
    finally:
        ctx.forget_runs(runs)


@pytest.mark.parametrize("name", sorted(DOC["cases"]))
def test_hand_worked_leak_cases(ctx, name):
    """O6 / O8 hand-worked cases through the library: every field of every leak row."""
    case = DOC["cases"][name]
    got = _compare_invocations(ctx, H.golden_case_invocations(case))
    H.assert_leaks_equal_golden(got, case)


def test_myers_examples(ctx):
    """Appendix A M1-M3 as evidences: the second run of a class is aligned against the first."""
    doc = H.load_golden("myers_examples.json")
    kid = {k: 100 + i for i, k in enumerate("ABCDE")}
    body = [[0, [[0, 8, 64]]]]
    for case in doc["cases"]:
        invs = []
        for run, seq_names in ((0, case["evidence"]), (2, case["run"])):
            for q, nm in enumerate(seq_names):
                invs.append((run, 0, q, 1, kid[nm], H.dsl_records(body, 1)))
        invs.append((1, 1, 0, 1, kid["A"], H.dsl_records(body, 1)))
        _ingest_invocations(ctx, invs)
        try:
            g = ctx.build([0, 2])
            blob = H.parse_blob(g.export())
            assert [int(k) for k in blob["slots"]["kernel_id"]] == [kid[k] for k in case["order_kernels"]], case["id"]
            got_counts = [int(c) for c in blob["slots"]["count"]]
            if "slot_counts" in case:
                assert got_counts == case["slot_counts"], case["id"]
            else:
                assert got_counts == [case["counts"][k] for k in case["order_kernels"]], case["id"]
        finally:
            ctx.forget_runs([0, 1, 2])


def _random_sequence_case(rng):
    """Runs of both classes, each launching a random kernel sequence over {A, B, C} (repeats, insertions and
    deletions anywhere); every invocation's records depend on (kernel, class) so CF / DF tests exist, and a
    per-run extra access makes some attributes differ across runs."""
    kid = {0: 0xA0, 1: 0xB0, 2: 0xC0}
    base = [int(x) for x in rng.integers(0, 3, size=int(rng.integers(1, 6)))]
    invs = []
    runs = int(rng.integers(2, 9))
    for run in range(runs):
        cls = run & 1
        seq = list(base)
        for _ in range(int(rng.integers(0, 3))):  # edits: insert / delete / replace at a random position
            op = int(rng.integers(0, 3))
            pos = int(rng.integers(0, len(seq) + 1))
            if op == 0 or not seq:
                seq.insert(pos, int(rng.integers(0, 3)))
            elif op == 1 and len(seq) > 1:
                del seq[min(pos, len(seq) - 1)]
            else:
                seq[min(pos, len(seq) - 1)] = int(rng.integers(0, 3))
        for q, k in enumerate(seq):
            nw = 1 + k
            lanes = 8 + 8 * cls if k != 2 else 16
            visits = [[k, [[0, lanes, 64 * k + 4096 * cls * (k == 0)]]],
                      [3 + (cls if k == 1 else 0), [[1, 4 + (run % 3), 512]]]]
            invs.append((run, cls, q, nw, kid[k], H.dsl_records(visits, nw)))
    return invs


def test_random_kernel_sequences(ctx):
    """200 random multi-run cases (Myers on repeated ids / mid-sequence edits, kernel leaks, slot ids that do not
    follow the alignment): evidences, KS rows, leaks and diff rows equal the oracle's."""
    rng = np.random.default_rng(20240)
    n_kernel_leaks = n_shifted = 0
    for _ in range(200):
        invs = _random_sequence_case(rng)
        if len({i[1] for i in invs}) < 2:
            continue
        gl = _compare_invocations(ctx, invs)
        n_kernel_leaks += int(np.sum(gl["kind"] == 0))
        n_shifted += int(np.sum((gl["kind"] != 0) & (gl["slot_fix"] != gl["slot_rnd"])))
    assert n_kernel_leaks > 50 and n_shifted > 10, (n_kernel_leaks, n_shifted)


@pytest.mark.parametrize("div,nf,nr", [(16, 4, 4), (4, 3, 5)])
def test_kernel_sequence_config_parity(ctx, div, nf, nr):
    """tracegen config 9 (secret-dependent launch sequence E L [G] L [G] L [L] [N] over the C4 kernel bodies)."""
    p = tracegen.Params.preset(9, grid_div=div, runs_fix=nf, runs_rnd=nr)
    ef, er, of, orr = _build_and_compare(ctx, p)
    assert ef.info()["n_slots"] >= 6
