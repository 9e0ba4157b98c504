"""B200-native TGOpt hot path: redundancy-aware batched TGAT inference.

The product is libtg.so (hand-written sm_100a CUDA behind the C ABI in
include/tg.h); `tg` is its thin ctypes binding. No CPU fallback exists.
"""
from .tg import (Context, TGError, lib, version, counters_dict,  # noqa: F401
                 TG_OPT_DEDUP, TG_OPT_CACHE, TG_OPT_TTABLE, TG_OPT_ALL, TG_OPT_HOST_CACHE,
                 TG_PREC_FP32, TG_PREC_TF32X3, TG_PREC_BF16, TG_PREC_TF32, TG_PREC_F16X3, TG_NCOUNTERS)
