"""Seeded synthetic trace generator (TEST / BENCH INFRASTRUCTURE, shared by the oracle and the CUDA path).

Stands in for Owl's tracers (NVBit + Pin; out of scope).  It holds none of the method's
arithmetic: it only says which warp entered which basic block and which thread touched which address.
The recipe of each workload is in owl_gen_core.h and DESIGN.md §4.  Host generation (libowlgen.so) feeds
the CPU oracle; device generation (libowlgen_cuda.so) writes the same bytes straight into HBM.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
MASTER_SEED = 0x4F574C21

RECORD_DTYPE = np.dtype([("addr", "<u8"), ("gwarp", "<u4"), ("meta", "<u4")])
FIX, RND = 0, 1

# Paper-shaped configurations (BASELINE.json configs[0..4]).
CONFIGS = {
    1: dict(runs_fix=10, runs_rnd=10, grid_div=1),     # toy: 1 kernel, 256 threads, 2 x 10 runs
    2: dict(runs_fix=100, runs_rnd=100, grid_div=1),   # AES-128 T-table, 64K threads
    3: dict(runs_fix=100, runs_rnd=100, grid_div=1),   # RSA modexp, 4K threads
    4: dict(runs_fix=50, runs_rnd=50, grid_div=1),     # PyTorch-shaped ops
    5: dict(runs_fix=500, runs_rnd=500, grid_div=1),   # nvJPEG-shaped decode, 1000 runs
    # RQ2 trace-size sweep (Fig. 5): threads = the input size
    6: dict(runs_fix=1, runs_rnd=0, grid_div=1, threads=1024),  # pattern 2: dummy S-box program
    7: dict(runs_fix=1, runs_rnd=0, grid_div=1, threads=1024),  # pattern 3: thread-distinct pixels
    8: dict(runs_fix=1, runs_rnd=0, grid_div=1, threads=1024),  # pattern 1: fixed threads
    # kernel-sequence model (Myers on repeated kernel ids, mid-sequence insertions / deletions)
    9: dict(runs_fix=8, runs_rnd=8, grid_div=1),
}
CONFIG_NAMES = {1: "C1-toy", 2: "C2-aes128-ttable", 3: "C3-rsa-modexp", 4: "C4-pytorch-ops", 5: "C5-nvjpeg-decode",
                6: "RQ2-sbox", 7: "RQ2-pixel", 8: "RQ2-fixed-threads", 9: "C9-kernel-sequence-model"}


class _Params(ctypes.Structure):
    _fields_ = [("config", ctypes.c_uint32), ("grid_div", ctypes.c_uint32), ("runs_fix", ctypes.c_uint32),
                ("runs_rnd", ctypes.c_uint32), ("seed", ctypes.c_uint64), ("threads", ctypes.c_uint32),
                ("_pad", ctypes.c_uint32)]


@dataclass(frozen=True)
class Params:
    config: int
    runs_fix: int
    runs_rnd: int
    grid_div: int = 1
    seed: int = MASTER_SEED
    threads: int = 0

    @staticmethod
    def preset(config: int, **over) -> "Params":
        kw = dict(CONFIGS[config])
        kw.update(over)
        return Params(config=config, **kw)

    def c(self) -> _Params:
        return _Params(self.config, self.grid_div, self.runs_fix, self.runs_rnd, self.seed, self.threads, 0)

    @property
    def n_runs(self) -> int:
        return self.runs_fix + self.runs_rnd


_host = None
_dev = None


def _load_host():
    global _host
    if _host is None:
        lib = ctypes.CDLL(os.path.join(_HERE, "libowlgen.so"))
        P = ctypes.POINTER(_Params)
        u32, u64 = ctypes.c_uint32, ctypes.c_uint64
        lib.ogh_run_class.argtypes = [P, u32]; lib.ogh_run_class.restype = u32
        lib.ogh_n_seq.argtypes = [P, u32]; lib.ogh_n_seq.restype = u32
        lib.ogh_seq_meta.argtypes = [P, u32, u32, ctypes.POINTER(u64), ctypes.POINTER(u32), ctypes.POINTER(u32)]
        lib.ogh_seq_meta.restype = None
        lib.ogh_seq_count.argtypes = [P, u32, u32, ctypes.c_void_p, ctypes.c_int]; lib.ogh_seq_count.restype = u64
        lib.ogh_seq_generate.argtypes = [P, u32, u32, ctypes.c_void_p, ctypes.c_int]
        lib.ogh_seq_generate.restype = u64
        _host = lib
    return _host


def _load_dev():
    global _dev
    if _dev is None:
        lib = ctypes.CDLL(os.path.join(_HERE, "libowlgen_cuda.so"))
        P = ctypes.POINTER(_Params)
        u32 = ctypes.c_uint32
        lib.ogd_seq_offsets.argtypes = [P, u32, u32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.ogd_seq_offsets.restype = ctypes.c_int
        lib.ogd_seq_generate.argtypes = [P, u32, u32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.ogd_seq_generate.restype = ctypes.c_int
        _dev = lib
    return _dev


@dataclass
class SegmentMeta:
    run: int
    input_class: int
    seq: int
    n_warps: int
    kernel_id: int


def run_class(p: Params, run: int) -> int:
    pc = p.c()
    return int(_load_host().ogh_run_class(ctypes.byref(pc), run))


def run_segments(p: Params, run: int) -> list[SegmentMeta]:
    lib = _load_host()
    pc = p.c()
    out = []
    for s in range(lib.ogh_n_seq(ctypes.byref(pc), run)):
        kid, nw, cls = ctypes.c_uint64(), ctypes.c_uint32(), ctypes.c_uint32()
        lib.ogh_seq_meta(ctypes.byref(pc), run, s, ctypes.byref(kid), ctypes.byref(nw), ctypes.byref(cls))
        out.append(SegmentMeta(run, int(cls.value), s, int(nw.value), int(kid.value)))
    return out


def host_count(p: Params, run: int, seq: int, threads: int = 0) -> int:
    pc = p.c()
    return int(_load_host().ogh_seq_count(ctypes.byref(pc), run, seq, None, threads or os.cpu_count() or 1))


def host_records(p: Params, run: int, seq: int, threads: int = 0) -> np.ndarray:
    """Warp-major records of one kernel invocation, as a numpy structured array (RECORD_DTYPE)."""
    lib = _load_host()
    pc = p.c()
    th = threads or os.cpu_count() or 1
    n = int(lib.ogh_seq_count(ctypes.byref(pc), run, seq, None, th))
    rec = np.empty(n, dtype=RECORD_DTYPE)
    got = int(lib.ogh_seq_generate(ctypes.byref(pc), run, seq, rec.ctypes.data, th))
    assert got == n
    return rec


def device_records(p: Params, run: int, seq: int, device=None, stream=None):
    """Generates the same records on the GPU; returns a torch uint8 tensor of 16*n bytes on `device`."""
    import torch
    lib = _load_dev()
    pc = p.c()
    meta = run_segments(p, run)[seq]
    dev = torch.device(device if device is not None else "cuda")
    st = stream if stream is not None else torch.cuda.current_stream(dev)
    counts = torch.empty(meta.n_warps, dtype=torch.int64, device=dev)
    offs = torch.empty(meta.n_warps + 1, dtype=torch.int64, device=dev)
    err = lib.ogd_seq_offsets(ctypes.byref(pc), run, seq, counts.data_ptr(), offs.data_ptr(), st.cuda_stream)
    if err:
        raise RuntimeError(f"ogd_seq_offsets: cuda error {err}")
    n = int(offs[-1].item())
    buf = torch.empty(max(n, 1) * 16, dtype=torch.uint8, device=dev)
    err = lib.ogd_seq_generate(ctypes.byref(pc), run, seq, offs.data_ptr(), buf.data_ptr(), st.cuda_stream)
    if err:
        raise RuntimeError(f"ogd_seq_generate: cuda error {err}")
    return buf[: n * 16], n


def device_interleave(buf, n: int, burst: int = 32):
    """Channel-order variant of a warp-major device buffer (same order as interleave(): bursts of `burst` records
    per warp, warps round-robin), built with torch on the device (bench / test infrastructure).  Returns a new
    uint8 tensor of 16*n bytes."""
    import torch
    if n == 0:
        return buf.clone()
    rec = buf[: n * 16].view(torch.int32).view(n, 4)
    g = rec[:, 2].to(torch.int64) & 0xFFFFFFFF
    pos = torch.arange(n, device=buf.device, dtype=torch.int64)
    first = torch.ones(n, dtype=torch.bool, device=buf.device)
    first[1:] = g[1:] != g[:-1]
    start = torch.cummax(torch.where(first, pos, torch.zeros_like(pos)), 0).values  # start of each record's warp
    q = (pos - start) // burst
    order = torch.argsort(q * (1 << 33) + start, stable=True)  # round q, then the warps in stream order
    return rec[order].contiguous().view(torch.uint8).view(-1)


def interleave(rec: np.ndarray, burst: int = 32) -> np.ndarray:
    """Channel-order variant (reading R17): bursts of `burst` records per warp, warps round-robin.
    Pure reordering: each warp's records keep their relative order."""
    if len(rec) == 0:
        return rec.copy()
    g = rec["gwarp"]
    starts = np.flatnonzero(np.r_[True, g[1:] != g[:-1]])
    ends = np.r_[starts[1:], len(rec)]
    pieces = []
    pos = starts.copy()
    while True:
        live = pos < ends
        if not live.any():
            break
        for i in np.flatnonzero(live):
            e = min(pos[i] + burst, ends[i])
            pieces.append(rec[pos[i]:e])
            pos[i] = e
    return np.concatenate(pieces)
