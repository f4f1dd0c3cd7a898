"""N1 input-class filtering (§VI) in the oracle, pinned by how the inputs were made: runs
replaying one secret give identical traces (one class), distinct secrets give distinct traces, and a
single changed record splits a class."""
import numpy as np

import tracegen
from oracle import oracle
from tests import helpers as H


def _by_run(p, runs):
    out = []
    for r in runs:
        segs = [oracle.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, tracegen.host_records(p, r, m.seq))
                for m in tracegen.run_segments(p, r)]
        out.append((r, segs))
    return out


def test_fixed_secret_is_one_class_random_secrets_are_not():
    """C2 (AES T-table, secret = key, plaintexts fixed per thread): the FIX runs replay one key, so their
    traces are identical; every RND run draws its own key, so its T-table lookups differ."""
    p = tracegen.Params.preset(2, grid_div=64, runs_fix=3, runs_rnd=3)
    runs = list(range(p.n_runs))
    cls, n = oracle.filter_inputs(_by_run(p, runs))
    fix = [c for r, c in zip(runs, cls) if tracegen.run_class(p, r) == 0]
    rnd = [c for r, c in zip(runs, cls) if tracegen.run_class(p, r) == 1]
    assert len(set(fix)) == 1 and len(set(rnd)) == len(rnd) and not set(fix) & set(rnd)
    assert n == 1 + len(rnd)
    firsts = [c for i, c in enumerate(cls) if c not in cls[:i]]
    assert firsts == list(range(n))  # class ids in order of first appearance


def test_only_fixed_runs_means_leak_free_for_these_inputs():
    p = tracegen.Params.preset(2, grid_div=64, runs_fix=4, runs_rnd=0)
    cls, n = oracle.filter_inputs(_by_run(p, range(4)))
    assert n == 1 and cls == [0, 0, 0, 0]


def test_identical_copies_and_one_changed_record():
    rec = H.w1_records()
    other = rec.copy()
    i = int(np.flatnonzero(other["meta"] >> 31)[-1])  # the last MEM record: move its address
    other["addr"][i] = other["addr"][i] + np.uint64(4)
    runs = [(0, [oracle.Segment(0, 0, 0, 2, 10, rec)]), (1, [oracle.Segment(1, 1, 0, 2, 10, rec.copy())]),
            (2, [oracle.Segment(2, 0, 0, 2, 10, other)]), (3, [oracle.Segment(3, 0, 0, 2, 10, rec)])]
    cls, n = oracle.filter_inputs(runs)
    assert cls == [0, 0, 1, 0] and n == 2  # the input class given at ingest is ignored


def test_kernel_sequence_is_part_of_the_trace():
    """Same records, but one run launches the kernel under another call-stack id: different traces."""
    rec = H.w1_records()
    runs = [(0, [oracle.Segment(0, 0, 0, 2, 10, rec)]), (1, [oracle.Segment(1, 0, 0, 2, 11, rec)])]
    assert oracle.filter_inputs(runs) == ([0, 1], 2)


# ---- N4: the RQ2 trace-size workloads (Fig. 5) -------------------------------------------------

def _rq2(cfg, threads):
    import struct
    p = tracegen.Params.preset(cfg, threads=threads)
    segs = [oracle.Segment(0, m.input_class, m.seq, m.n_warps, m.kernel_id, tracegen.host_records(p, 0, m.seq))
            for m in tracegen.run_segments(p, 0)]
    blob = oracle.build(segs).export()
    return sum(len(s.records) for s in segs), struct.unpack_from("<4Q", blob, 24)


def test_rq2_growth_patterns():
    """The three growth patterns of P:L366 as closed forms of the workloads' construction: (1) fixed threads:
    records and cells constant; (2) S-box lookups: records grow linearly, address cells saturate at 16 x 256;
    (3) thread-distinct pixels: cells = 5 per thread.  Records = accesses + one BB entry per traced warp."""
    for t in (100, 777, 4096):
        warps = -(-t // 32)
        rec2, cells2 = _rq2(6, t)
        rec3, cells3 = _rq2(7, t)
        rec1, cells1 = _rq2(8, t)
        assert rec2 == 16 * t + warps and cells2[3] <= 16 * 256
        assert rec3 == 5 * t + warps and cells3[3] == 5 * t
        assert rec1 == 8 * 256 + 8 and cells1[3] == 64
        assert cells1[:3] == cells2[:3] == cells3[:3] == (1, 2, 1)  # one BB: node, S->B0, B0->S, one triple
    assert _rq2(6, 20000)[1][3] == 16 * 256  # saturated
