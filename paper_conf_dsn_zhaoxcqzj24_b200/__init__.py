"""B200-native hot path of Owl's differential side-channel detector (Zhao et al., DSN 2024).

The product is libowl.so (C ABI in include/owl.h, CUDA kernels for sm_100a in csrc/).  This package is the
thin Python binding over it (ctypes; argument marshalling only) plus the multi-GPU orchestration through
torch.distributed.  There is no CPU fallback: importing the binding fails loudly when libowl.so is missing.
"""
from .api import (Adcfg, Context, OwlError, Segment, DIFF_DTYPE, KS_DTYPE, LEAK_DTYPE,  # noqa: F401
                  OWL_FIXED, OWL_RANDOM, OWL_SEG_WARP_MAJOR, OWL_SEG_HOST_RECORDS, version)
