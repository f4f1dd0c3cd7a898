"""Python binding of libowl (same names as include/owl.h; argument marshalling only).

    ctx = Context(device)                         # owl_ctx_create
    ctx.ingest([Segment(...), ...], stream)       # owl_ingest_traces   (A1)
    ef = ctx.build(runs_fix); er = ctx.build(runs_rnd)   # owl_build_adcfg (A2-A4)
    rows = ctx.diff(a, b)                         # owl_diff_adcfg      (A5)
    leaks = ctx.leak_test(ef, er, 0.05)           # owl_leak_test       (A6-A7)

Every step of the path runs inside libowl's CUDA kernels; PyTorch only provides device memory and streams.
"""
from __future__ import annotations

import ctypes
import weakref

import numpy as np

from . import _lib

OWL_FIXED, OWL_RANDOM = 0, 1
OWL_SEG_WARP_MAJOR, OWL_SEG_HOST_RECORDS = 1, 2
OWL_CHANNEL_AUTO, OWL_CHANNEL_COPY, OWL_CHANNEL_IN_PLACE = 0, 1, 2  # owl_config.channel_order (N2)

DIFF_DTYPE = np.dtype([("table", "<u4"), ("slot", "<u4"), ("bb", "<u4"), ("ins", "<u4"), ("j", "<u4"),
                       ("prev", "<u4"), ("next", "<u4"), ("_pad", "<u4"), ("x", "<u8"), ("count_a", "<u8"),
                       ("count_b", "<u8")])
LEAK_DTYPE = np.dtype([("kind", "<u4"), ("slot_fix", "<u4"), ("slot_rnd", "<u4"), ("bb", "<u4"), ("ins", "<u4"),
                       ("j", "<u4"), ("kernel_id", "<u8"), ("n", "<u8"), ("m", "<u8"), ("K_lo", "<u8"),
                       ("K_hi", "<u8"), ("D", "<f8"), ("p", "<f8")])
KS_DTYPE = np.dtype([("kind", "<u4"), ("slot_fix", "<u4"), ("slot_rnd", "<u4"), ("bb", "<u4"), ("ins", "<u4"),
                     ("j", "<u4"), ("n", "<u8"), ("m", "<u8"), ("K_lo", "<u8"), ("K_hi", "<u8"), ("D", "<f8"),
                     ("p", "<f8"), ("fail", "<u4"), ("_pad", "<u4")])
STATUS = {0: "OWL_OK", 1: "OWL_ERR_INVALID_ARG", 2: "OWL_ERR_MALFORMED_TRACE", 3: "OWL_ERR_OUT_OF_MEMORY",
          4: "OWL_ERR_CUDA", 5: "OWL_ERR_NCCL", 6: "OWL_ERR_STATE", 7: "OWL_ERR_CAPACITY"}


class OwlError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def _check(st):
    if st != 0:
        raise OwlError(st, _lib.load().owl_last_error().decode(errors="replace"))


def version() -> str:
    return _lib.load().owl_version().decode()


def _ptr(buf):
    """Device pointer of a torch tensor / host pointer of a numpy array."""
    if hasattr(buf, "data_ptr"):
        return buf.data_ptr()
    if isinstance(buf, np.ndarray):
        return buf.ctypes.data
    raise TypeError(type(buf))


class Segment:
    """One kernel invocation: metadata + a buffer of n 16-byte records (torch CUDA tensor, or a numpy array
    with flags |= OWL_SEG_HOST_RECORDS).  The buffer is kept alive by this object."""

    def __init__(self, run, input_class, seq, n_warps, kernel_id, buf, n_records, flags=OWL_SEG_WARP_MAJOR):
        self.run, self.input_class, self.seq, self.n_warps, self.kernel_id = run, input_class, seq, n_warps, kernel_id
        self.buf, self.n_records, self.flags = buf, int(n_records), flags
        if isinstance(buf, np.ndarray):
            self.flags |= OWL_SEG_HOST_RECORDS

    def c(self):
        return _lib.OwlSegment(self.run, self.input_class, self.seq, self.n_warps, self.kernel_id, self.n_records,
                               _ptr(self.buf) if self.n_records else None, self.flags, 0)


def _u32arr(xs):
    xs = list(xs)
    return (ctypes.c_uint32 * max(1, len(xs)))(*xs), len(xs)


def _take(ptr, n, dtype):
    L = _lib.load()
    if n == 0:
        if ptr.value:
            L.owl_free(ptr)
        return np.zeros(0, dtype=dtype)
    # zero-copy: the array views the library's malloc'd rows and frees them when it is collected
    buf = (ctypes.c_char * (n * dtype.itemsize)).from_address(ptr.value)
    out = np.frombuffer(buf, dtype=dtype)
    weakref.finalize(buf, L.owl_free, ctypes.c_void_p(ptr.value))
    return out


class Adcfg:
    """A device-resident A-DCFG (one run) or class evidence (owl_adcfg*)."""

    def __init__(self, ctx, h):
        self.ctx, self.h = ctx, h

    def __del__(self):
        self.destroy()

    def destroy(self):
        if getattr(self, "h", None):
            _lib.load().owl_adcfg_destroy(self.h)
            self.h = None

    def export(self, path=None) -> bytes:
        blob, n = ctypes.c_void_p(), ctypes.c_size_t()
        _check(_lib.load().owl_adcfg_export(self.h, path.encode() if path else None, ctypes.byref(blob), ctypes.byref(n)))
        data = ctypes.string_at(blob.value, n.value)
        _lib.load().owl_free(blob)
        return data

    def info(self):
        i = _lib.OwlAdcfgInfo()
        _check(_lib.load().owl_adcfg_info_get(self.h, ctypes.byref(i)))
        return dict(input_class=i.input_class, n_runs=i.n_runs, n_slots=i.n_slots, n_cells=list(i.n_cells),
                    n_records=i.n_records)

    def accumulate(self, runs):
        arr, n = _u32arr(runs)
        _check(_lib.load().owl_adcfg_accumulate(self.ctx.h, self.h, arr, n))

    def partition(self, world):
        """owl_partition_evidence: returns (device pointer, per-owner byte counts)."""
        ptr = ctypes.c_void_p()
        sb = (ctypes.c_uint64 * world)()
        _check(_lib.load().owl_partition_evidence(self.ctx.h, self.h, world, ctypes.byref(ptr), sb))
        return ptr.value, [int(x) for x in sb]


class Context:
    """owl_ctx: one per GPU / rank."""

    def __init__(self, device=0, config=None):
        L = _lib.load()
        h = ctypes.c_void_p()
        _check(L.owl_ctx_create(int(device), ctypes.byref(h)))
        self.h = h.value
        self.device = int(device)
        self._segs = {}
        self.stream = None
        if config:
            self.set_config(**config)

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:  # modules may be torn down at interpreter exit
            try:
                _lib.load().owl_ctx_destroy(self.h)
            except Exception:  # noqa: BLE001
                pass
            self.h = None

    def set_config(self, addr_capacity=0, cf_capacity=0, max_regrow=0, fold_ctas_per_sm=0, host_chunk_bytes=0,
                   hcf_reading=0, channel_order=0):
        """owl_ctx_set_config.  hcf_reading: 0 = joint counts (R1), 1 = row-normalized A (R2, Eq. 7).
        channel_order: 0 auto, 1 copy to warp-major, 2 fold in place through the burst index (include/owl.h)."""
        cfg = _lib.OwlConfig(addr_capacity, cf_capacity, max_regrow, fold_ctas_per_sm, host_chunk_bytes,
                             hcf_reading, channel_order)
        _check(_lib.load().owl_ctx_set_config(self.h, ctypes.byref(cfg)))

    def ingest(self, segments, stream=None):
        """owl_ingest_traces.  stream: a torch.cuda.Stream (default: the current stream)."""
        segments = list(segments)
        arr = (_lib.OwlSegment * max(1, len(segments)))(*[s.c() for s in segments])
        if stream is None:
            try:
                import torch
                stream = torch.cuda.current_stream(self.device)
            except Exception:  # noqa: BLE001
                stream = None
        sp = stream.cuda_stream if stream is not None else None
        _check(_lib.load().owl_ingest_traces(self.h, arr, len(segments), sp))
        for s in segments:
            self._segs[(s.run, s.seq)] = s
        self.stream = stream

    def forget_runs(self, runs):
        runs = list(runs)
        arr, n = _u32arr(runs)
        _check(_lib.load().owl_forget_runs(self.h, arr, n))
        for k in [k for k in self._segs if k[0] in set(runs)]:
            del self._segs[k]

    def register_remote_runs(self, runs, classes, seqs):
        """runs: run ids; classes: input class per run; seqs: list of kernel-id lists per run."""
        runs = list(runs)
        r = (ctypes.c_uint32 * max(1, len(runs)))(*runs)
        c = (ctypes.c_uint32 * max(1, len(runs)))(*classes)
        ln = (ctypes.c_uint32 * max(1, len(runs)))(*[len(s) for s in seqs])
        flat = [k for s in seqs for k in s]
        k = (ctypes.c_uint64 * max(1, len(flat)))(*flat)
        _check(_lib.load().owl_register_remote_runs(self.h, r, c, ln, k, len(runs)))

    def build(self, runs) -> Adcfg:
        arr, n = _u32arr(runs)
        h = ctypes.c_void_p()
        _check(_lib.load().owl_build_adcfg(self.h, arr, n, ctypes.byref(h)))
        return Adcfg(self, h.value)

    def diff(self, a: Adcfg, b: Adcfg) -> np.ndarray:
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        _check(_lib.load().owl_diff_adcfg(self.h, a.h, b.h, ctypes.byref(p), ctypes.byref(n)))
        return _take(p, n.value, DIFF_DTYPE)

    def filter_inputs(self, runs):
        """owl_filter_inputs (N1): (class of each run, number of classes); one class <=> the
        inputs show no trace difference.  Class ids in order of first appearance."""
        runs = list(runs)
        arr, n = _u32arr(runs)
        out = (ctypes.c_uint32 * max(1, n))()
        nc = ctypes.c_uint32()
        _check(_lib.load().owl_filter_inputs(self.h, arr, n, out, ctypes.byref(nc)))
        return np.array(out[:n], dtype=np.uint32), int(nc.value)

    def leak_test(self, e_fix: Adcfg, e_rnd: Adcfg, significance: float = 0.05) -> np.ndarray:
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        _check(_lib.load().owl_leak_test(self.h, e_fix.h, e_rnd.h, significance, ctypes.byref(p), ctypes.byref(n)))
        return _take(p, n.value, LEAK_DTYPE)

    def ks_tests(self, e_fix: Adcfg, e_rnd: Adcfg, significance: float = 0.05) -> np.ndarray:
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        _check(_lib.load().owl_ks_tests(self.h, e_fix.h, e_rnd.h, significance, ctypes.byref(p), ctypes.byref(n)))
        return _take(p, n.value, KS_DTYPE)

    def merge_leaks(self, e_fix: Adcfg, e_rnd: Adcfg, parts) -> np.ndarray:
        """owl_merge_leaks: the owners' leak rows (list of arrays) -> the one-GPU leak list."""
        rows = np.ascontiguousarray(np.concatenate(list(parts)) if len(parts) else np.zeros(0, LEAK_DTYPE),
                                    dtype=LEAK_DTYPE)
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        _check(_lib.load().owl_merge_leaks(self.h, e_fix.h, e_rnd.h, rows.ctypes.data if len(rows) else None,
                                           len(rows), ctypes.byref(p), ctypes.byref(n)))
        return _take(p, n.value, LEAK_DTYPE)

    def merge_diffs(self, a: Adcfg, b: Adcfg, parts) -> np.ndarray:
        """owl_merge_diffs: the owners' diff rows (list of arrays) -> canonical order, slot rows once."""
        rows = np.ascontiguousarray(np.concatenate(list(parts)) if len(parts) else np.zeros(0, DIFF_DTYPE),
                                    dtype=DIFF_DTYPE)
        p, n = ctypes.c_void_p(), ctypes.c_size_t()
        _check(_lib.load().owl_merge_diffs(self.h, a.h, b.h, rows.ctypes.data if len(rows) else None, len(rows),
                                           ctypes.byref(p), ctypes.byref(n)))
        return _take(p, n.value, DIFF_DTYPE)

    def absorb(self, like: Adcfg, recv_ptr, recv_bytes, rank) -> Adcfg:
        world = len(recv_bytes)
        rb = (ctypes.c_uint64 * world)(*recv_bytes)
        h = ctypes.c_void_p()
        _check(_lib.load().owl_absorb_evidence(self.h, like.h, recv_ptr, rb, world, rank, ctypes.byref(h)))
        return Adcfg(self, h.value)

    def stats(self):
        fl, lr, tr = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
        lm, tm = ctypes.c_double(), ctypes.c_double()
        _check(_lib.load().owl_get_stats(self.h, ctypes.byref(fl), ctypes.byref(lm), ctypes.byref(lr),
                                         ctypes.byref(tm), ctypes.byref(tr)))
        return dict(fold_launches=fl.value, last_fold_ms=lm.value, last_fold_records=lr.value,
                    total_fold_ms=tm.value, total_fold_records=tr.value)

    def reset_stats(self):
        _check(_lib.load().owl_reset_stats(self.h))
