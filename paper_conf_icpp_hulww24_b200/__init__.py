"""B200-native engine for the AutoPipe partition cost model (Hu et al., ICPP '24).

The hot path — scoring pipeline partitions with the exact integer 1F1B cost model of SPEC.md — runs
in hand-written sm_100a CUDA kernels behind the C-ABI of include/autopipe.h; this package is the thin
Python binding (``Engine``) plus the multi-GPU driver (``distributed``). There is no CPU fallback.
"""
from ._lib import AutopipeError, USE_ALL_WORKERS, LIB_PATH  # noqa: F401  (raises if not built)
from .engine import Engine, SearchResult, U64_MAX, as_u64, reduce_results, result_from_bytes  # noqa: F401

__all__ = ["Engine", "SearchResult", "AutopipeError", "USE_ALL_WORKERS", "U64_MAX", "as_u64", "LIB_PATH",
           "reduce_results", "result_from_bytes"]
