"""ctypes declarations of libowl.so (include/owl.h).  Loading fails loudly if the library is missing."""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("OWL_LIBOWL_PATH") or os.path.join(_HERE, "libowl.so")

u32, u64, vp, sz = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_size_t


class OwlSegment(ctypes.Structure):
    _fields_ = [("run", u32), ("input_class", u32), ("seq", u32), ("n_warps", u32), ("kernel_id", u64),
                ("n_records", u64), ("records", vp), ("flags", u32), ("_reserved", u32)]


class OwlConfig(ctypes.Structure):
    _fields_ = [("addr_capacity", u64), ("cf_capacity", u64), ("max_regrow", u32), ("fold_ctas_per_sm", u32),
                ("host_chunk_bytes", u64), ("hcf_reading", u32), ("channel_order", u32)]


class OwlAdcfgInfo(ctypes.Structure):
    _fields_ = [("input_class", u32), ("n_runs", u32), ("n_slots", u32), ("_pad", u32), ("n_cells", u64 * 4),
                ("n_records", u64)]


# every symbol include/owl.h declares: name -> (restype, argtypes)
SIGNATURES = {
    "owl_ctx_create": (ctypes.c_int, [ctypes.c_int, ctypes.POINTER(vp)]),
    "owl_ctx_destroy": (ctypes.c_int, [vp]),
    "owl_ctx_set_config": (ctypes.c_int, [vp, ctypes.POINTER(OwlConfig)]),
    "owl_ingest_traces": (ctypes.c_int, [vp, ctypes.POINTER(OwlSegment), sz, vp]),
    "owl_forget_runs": (ctypes.c_int, [vp, ctypes.POINTER(u32), sz]),
    "owl_build_adcfg": (ctypes.c_int, [vp, ctypes.POINTER(u32), sz, ctypes.POINTER(vp)]),
    "owl_adcfg_accumulate": (ctypes.c_int, [vp, vp, ctypes.POINTER(u32), sz]),
    "owl_adcfg_info_get": (ctypes.c_int, [vp, ctypes.POINTER(OwlAdcfgInfo)]),
    "owl_adcfg_export": (ctypes.c_int, [vp, ctypes.c_char_p, ctypes.POINTER(vp), ctypes.POINTER(sz)]),
    "owl_adcfg_destroy": (ctypes.c_int, [vp]),
    "owl_diff_adcfg": (ctypes.c_int, [vp, vp, vp, ctypes.POINTER(vp), ctypes.POINTER(sz)]),
    "owl_filter_inputs": (ctypes.c_int, [vp, ctypes.POINTER(u32), sz, ctypes.POINTER(u32), ctypes.POINTER(u32)]),
    "owl_leak_test": (ctypes.c_int, [vp, vp, vp, ctypes.c_double, ctypes.POINTER(vp), ctypes.POINTER(sz)]),
    "owl_ks_tests": (ctypes.c_int, [vp, vp, vp, ctypes.c_double, ctypes.POINTER(vp), ctypes.POINTER(sz)]),
    "owl_partition_evidence": (ctypes.c_int, [vp, vp, ctypes.c_int, ctypes.POINTER(vp), ctypes.POINTER(u64)]),
    "owl_absorb_evidence": (ctypes.c_int, [vp, vp, vp, ctypes.POINTER(u64), ctypes.c_int, ctypes.c_int,
                                           ctypes.POINTER(vp)]),
    "owl_merge_leaks": (ctypes.c_int, [vp, vp, vp, vp, sz, ctypes.POINTER(vp), ctypes.POINTER(sz)]),
    "owl_merge_diffs": (ctypes.c_int, [vp, vp, vp, vp, sz, ctypes.POINTER(vp), ctypes.POINTER(sz)]),
    "owl_register_remote_runs": (ctypes.c_int, [vp, ctypes.POINTER(u32), ctypes.POINTER(u32), ctypes.POINTER(u32),
                                                ctypes.POINTER(u64), sz]),
    "owl_get_stats": (ctypes.c_int, [vp, ctypes.POINTER(u64), ctypes.POINTER(ctypes.c_double), ctypes.POINTER(u64),
                                     ctypes.POINTER(ctypes.c_double), ctypes.POINTER(u64)]),
    "owl_reset_stats": (ctypes.c_int, [vp]),
    "owl_free": (None, [vp]),
    "owl_last_error": (ctypes.c_char_p, []),
    "owl_version": (ctypes.c_char_p, []),
}

_lib = None


def load():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"libowl.so not found at {LIB_PATH}: run `python __graft_entry__.py` (build) first; "
                              "there is no CPU fallback")
        lib = ctypes.CDLL(LIB_PATH)
        lenient = os.environ.get("OWL_LIB_LENIENT") == "1"  # experiments: older library builds
        for name, (res, args) in SIGNATURES.items():
            if lenient and not hasattr(lib, name):
                continue
            fn = getattr(lib, name)
            fn.restype = res
            fn.argtypes = args
        _lib = lib
    return _lib
