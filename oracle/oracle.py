"""ctypes wrapper of the CPU oracle (liboracle.so).  TEST INFRASTRUCTURE ONLY.

May be imported only by tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
legs; the product package never imports it (tests/test_abi.py checks that).  See owl_oracle.cpp for what
it computes and which paper passage each step follows.
"""
from __future__ import annotations

import ctypes
import os
import time

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))

DIFF_DTYPE = np.dtype([("table", "<u4"), ("slot", "<u4"), ("bb", "<u4"), ("ins", "<u4"), ("j", "<u4"),
                       ("prev", "<u4"), ("next", "<u4"), ("_pad", "<u4"), ("x", "<u8"), ("count_a", "<u8"),
                       ("count_b", "<u8")])
LEAK_DTYPE = np.dtype([("kind", "<u4"), ("slot_fix", "<u4"), ("slot_rnd", "<u4"), ("bb", "<u4"), ("ins", "<u4"),
                       ("j", "<u4"), ("kernel_id", "<u8"), ("n", "<u8"), ("m", "<u8"), ("K_lo", "<u8"),
                       ("K_hi", "<u8"), ("D", "<f8"), ("p", "<f8")])
KS_DTYPE = np.dtype([("kind", "<u4"), ("slot_fix", "<u4"), ("slot_rnd", "<u4"), ("bb", "<u4"), ("ins", "<u4"),
                     ("j", "<u4"), ("n", "<u8"), ("m", "<u8"), ("K_lo", "<u8"), ("K_hi", "<u8"), ("D", "<f8"),
                     ("p", "<f8"), ("fail", "<u4"), ("_pad", "<u4")])


class _Seg(ctypes.Structure):
    _fields_ = [("run", ctypes.c_uint32), ("input_class", ctypes.c_uint32), ("seq", ctypes.c_uint32),
                ("n_warps", ctypes.c_uint32), ("kernel_id", ctypes.c_uint64), ("n_records", ctypes.c_uint64),
                ("records", ctypes.c_void_p)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = bind(ctypes.CDLL(os.path.join(_HERE, "liboracle.so")))
    return _lib


def bind(L):
    """Declares the C signatures on a loaded oracle library (also used by the mutation tests, which load
    deliberately broken builds of owl_oracle.cpp to show that the pins catch them)."""
    vp, sz = ctypes.c_void_p, ctypes.c_size_t
    L.orc_build.argtypes = [ctypes.POINTER(_Seg), sz, ctypes.c_int]; L.orc_build.restype = vp
    L.orc_free.argtypes = [vp]; L.orc_free.restype = None
    L.orc_last_error.restype = ctypes.c_char_p
    L.orc_export.argtypes = [vp, vp, sz]; L.orc_export.restype = sz
    L.orc_diff.argtypes = [vp, vp, vp, sz]; L.orc_diff.restype = sz
    L.orc_ks_tests.argtypes = [vp, vp, ctypes.c_double, vp, sz]; L.orc_ks_tests.restype = sz
    L.orc_leak_test.argtypes = [vp, vp, ctypes.c_double, vp, sz]; L.orc_leak_test.restype = sz
    L.orc_myers.argtypes = [vp, sz, vp, sz, vp, sz]; L.orc_myers.restype = sz
    L.orc_ks_hist.argtypes = [vp, vp, sz, vp, vp, sz, ctypes.c_double, vp]; L.orc_ks_hist.restype = None
    L.orc_slots.argtypes = [vp, vp, vp, vp, sz]; L.orc_slots.restype = sz
    L.orc_evidence_new.argtypes = [ctypes.c_uint32]; L.orc_evidence_new.restype = vp
    L.orc_evidence_add.argtypes = [vp, ctypes.POINTER(_Seg), sz, ctypes.c_int]; L.orc_evidence_add.restype = ctypes.c_int
    return L


class OracleError(RuntimeError):
    pass


class Segment:
    """One kernel invocation for the oracle: metadata + host records (numpy, 16-byte records)."""

    def __init__(self, run, input_class, seq, n_warps, kernel_id, records):
        self.run, self.input_class, self.seq, self.n_warps, self.kernel_id = run, input_class, seq, n_warps, kernel_id
        self.records = np.ascontiguousarray(records)


class Adcfg:
    def __init__(self, h):
        self.h = h

    def __del__(self):
        if getattr(self, "h", None):
            lib().orc_free(self.h)
            self.h = None

    def export(self) -> bytes:
        n = lib().orc_export(self.h, None, 0)
        buf = ctypes.create_string_buffer(n)
        lib().orc_export(self.h, buf, n)
        return buf.raw

    def slots(self):
        n = lib().orc_slots(self.h, None, None, None, 0)
        s = np.empty(n, np.uint32); k = np.empty(n, np.uint64); c = np.empty(n, np.uint64)
        lib().orc_slots(self.h, s.ctypes.data, k.ctypes.data, c.ctypes.data, n)
        return s, k, c


def build(segments, threads: int = 0) -> Adcfg:
    """O1-O4: per-run A-DCFGs merged into one evidence (one input class)."""
    arr = (_Seg * max(1, len(segments)))()
    for i, s in enumerate(segments):
        arr[i] = _Seg(s.run, s.input_class, s.seq, s.n_warps, s.kernel_id, len(s.records),
                      s.records.ctypes.data if len(s.records) else None)
    h = lib().orc_build(arr, len(segments), threads)
    if not h:
        raise OracleError(lib().orc_last_error().decode())
    return Adcfg(h)


class Evidence(Adcfg):
    """An evidence built incrementally (O1-O4 over batches of runs merged in ascending run order): the same
    result as build() over all the runs, for workloads larger than host memory."""

    def __init__(self, input_class: int):
        super().__init__(lib().orc_evidence_new(input_class))

    def add(self, segments, threads: int = 0):
        arr = (_Seg * max(1, len(segments)))()
        for i, s in enumerate(segments):
            arr[i] = _Seg(s.run, s.input_class, s.seq, s.n_warps, s.kernel_id, len(s.records),
                          s.records.ctypes.data if len(s.records) else None)
        if lib().orc_evidence_add(self.h, arr, len(segments), threads) != 0:
            raise OracleError(lib().orc_last_error().decode())


def _rows(fn, dtype, *args):
    n = fn(*args, None, 0)
    out = np.zeros(n, dtype=dtype)
    if n:
        fn(*args, out.ctypes.data, n)
    return out


def diff(a: Adcfg, b: Adcfg) -> np.ndarray:
    return _rows(lib().orc_diff, DIFF_DTYPE, a.h, b.h)


def ks_tests(f: Adcfg, r: Adcfg, significance: float = 0.05) -> np.ndarray:
    return _rows(lib().orc_ks_tests, KS_DTYPE, f.h, r.h, significance)


def leak_test(f: Adcfg, r: Adcfg, significance: float = 0.05) -> np.ndarray:
    return _rows(lib().orc_leak_test, LEAK_DTYPE, f.h, r.h, significance)


def myers(a, b):
    a = np.asarray(a, dtype=np.uint64); b = np.asarray(b, dtype=np.uint64)
    n = lib().orc_myers(a.ctypes.data, len(a), b.ctypes.data, len(b), None, 0)
    out = np.zeros(3 * max(n, 1), dtype=np.int32)
    lib().orc_myers(a.ctypes.data, len(a), b.ctypes.data, len(b), out.ctypes.data, 3 * n)
    names = {0: "M", 1: "D", 2: "I"}
    return [(names[int(out[3 * i])], int(out[3 * i + 1]), int(out[3 * i + 2])) for i in range(n)]


def ks_hist(xf, cf, xr, cr, significance: float = 0.05):
    xf = np.asarray(xf, np.uint64); cf = np.asarray(cf, np.uint64)
    xr = np.asarray(xr, np.uint64); cr = np.asarray(cr, np.uint64)
    out = np.zeros(1, dtype=KS_DTYPE)
    lib().orc_ks_hist(xf.ctypes.data, cf.ctypes.data, len(xf), xr.ctypes.data, cr.ctypes.data, len(xr),
                      significance, out.ctypes.data)
    return out[0]


def run_config(params, runs=None, threads: int = 0):
    """Convenience for tests / bench: host-generate the runs of a tracegen config and build E_fix, E_rnd."""
    import tracegen
    runs = list(range(params.n_runs)) if runs is None else list(runs)
    by_cls = {0: [], 1: []}
    t_gen = time.perf_counter()
    for r in runs:
        for m in tracegen.run_segments(params, r):
            rec = tracegen.host_records(params, r, m.seq, threads)
            by_cls[m.input_class].append(Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, rec))
    t_gen = time.perf_counter() - t_gen
    return by_cls, t_gen


def filter_inputs(segments_by_run, threads: int = 0):
    """N1, input-class filtering (§VI): "inputs that generate identical traces [are] the same
    class".  The plain definition: build each run's A-DCFG (its segments, one input class for all) and
    group the runs whose canonical dumps are byte-identical, classes numbered in order of first
    appearance.  segments_by_run: list of (run, [Segment]) in the order to visit.  Returns
    (class_of list, n_classes)."""
    seen, class_of = {}, []
    for run, segs in segments_by_run:
        same_class = [Segment(s.run, 0, s.seq, s.n_warps, s.kernel_id, s.records) for s in segs]
        blob = build(same_class, threads).export()
        class_of.append(seen.setdefault(blob, len(seen)))
    return class_of, len(seen)
