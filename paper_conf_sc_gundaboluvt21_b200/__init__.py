"""B200-native FastZ hot path: batched gapped y-drop seed extension (inspector -> binning -> trimmed
executor -> traceback) in hand-written sm_100a CUDA behind the C ABI of include/fastz.h.

The Python layer is a ctypes binding (``fastz``) plus the multi-GPU driver (``dist``); it never computes
any part of the method itself and never imports the CPU oracle.
"""
from .fastz import (Aligner, Alignments, FastzError, fastz_census, fastz_create, fastz_default_params,  # noqa: F401
                    fastz_destroy, fastz_extend_seeds, fastz_get_alignments, fastz_get_sides, fastz_get_stats,
                    fastz_int_peak, lib)
