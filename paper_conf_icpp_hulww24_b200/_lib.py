"""ctypes binding of the C-ABI in include/autopipe.h (argument marshalling only).

The shared library ``libautopipe.so`` is built in-tree by ``__graft_entry__.build()`` (nvcc,
sm_100a). There is no fallback: if the library is missing this module raises on import.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# AUTOPIPE_LIB may name another in-tree build of the same library (kernel-variant experiments)
LIB_PATH = os.environ.get("AUTOPIPE_LIB") or os.path.join(_HERE, "libautopipe.so")

AUTOPIPE_OK = 0
AUTOPIPE_E_INVAL = -1
AUTOPIPE_E_STATE = -2
AUTOPIPE_E_OVERFLOW = -3
AUTOPIPE_E_CUDA = -4
AUTOPIPE_E_NOMEM = -5
USE_ALL_WORKERS = 1
# row f3 (schedule variants, reading F-3)
SCHED_PIPEDREAM, SCHED_2BW, SCHED_GPIPE, SCHED_DAPPLE, SCHED_PIPEDREAM_RR, SCHED_CHIMERA = 0, 1, 2, 3, 4, 5
SYNC_RING, SYNC_PS = 0, 1
RECOMPUTE = 1
MAX_MICRO_BATCHES = 65536

ERROR_NAMES = {AUTOPIPE_E_INVAL: "AUTOPIPE_E_INVAL", AUTOPIPE_E_STATE: "AUTOPIPE_E_STATE",
               AUTOPIPE_E_OVERFLOW: "AUTOPIPE_E_OVERFLOW", AUTOPIPE_E_CUDA: "AUTOPIPE_E_CUDA",
               AUTOPIPE_E_NOMEM: "AUTOPIPE_E_NOMEM"}

# every symbol include/autopipe.h declares
SYMBOLS = ["autopipe_create", "autopipe_destroy", "autopipe_last_error", "autopipe_load_profile",
           "autopipe_set_state", "autopipe_set_state_device", "autopipe_eval_partitions", "autopipe_search_optimum",
           "autopipe_rollout_rewards", "autopipe_count_candidates", "autopipe_decode_index",
           "autopipe_int_path", "autopipe_kernel_launches", "autopipe_set_timing", "autopipe_set_search_options",
           "autopipe_last_search_ms", "autopipe_neighbourhood", "autopipe_neighbourhood_best",
           "autopipe_switch_rewards", "autopipe_balanced_shards", "autopipe_set_schedule",
           "autopipe_get_schedule", "autopipe_eval_partitions_w", "autopipe_rollout_rewards_w",
           "autopipe_search_optimum_w", "autopipe_decode_index_w", "autopipe_search_optimum_async",
           "autopipe_search_optimum_async_w", "autopipe_reduce_results", "autopipe_reduce_results_w", "autopipe_search_times",
           "autopipe_search_seed_async", "autopipe_set_search_bound", "autopipe_local_search",
           "autopipe_balanced_shards_path"]


class Partition(ctypes.Structure):
    _fields_ = [("n_stages", ctypes.c_uint8), ("last_layer", ctypes.c_uint8 * 7),
                ("stage_of_worker", ctypes.c_uint8 * 8)]


class Result(ctypes.Structure):
    _fields_ = [("time_ns", ctypes.c_uint64), ("index", ctypes.c_uint64),
                ("evaluated", ctypes.c_uint64), ("part", Partition)]


class PartitionW(ctypes.Structure):  # row f4: S <= 16 stages, N <= 16 workers
    _fields_ = [("n_stages", ctypes.c_uint8), ("last_layer", ctypes.c_uint8 * 15),
                ("stage_of_worker", ctypes.c_uint8 * 16)]


class ResultW(ctypes.Structure):
    _fields_ = [("time_ns", ctypes.c_uint64), ("index", ctypes.c_uint64),
                ("evaluated", ctypes.c_uint64), ("part", PartitionW)]


assert ctypes.sizeof(Partition) == 16 and ctypes.sizeof(Result) == 40
assert ctypes.sizeof(PartitionW) == 32 and ctypes.sizeof(ResultW) == 56


class AutopipeError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__("%s: %s" % (ERROR_NAMES.get(code, str(code)), msg))
        self.code = code


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError("libautopipe.so not built (run __graft_entry__.build()); there is no CPU "
                          "fallback for the cost-model kernels")
    lib = ctypes.CDLL(LIB_PATH)
    P = ctypes.c_void_p
    u32, u64, i32 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    pu64 = ctypes.POINTER(ctypes.c_uint64)
    sig = {
        "autopipe_create": (i32, [i32, ctypes.POINTER(P)]),
        "autopipe_destroy": (None, [P]),
        "autopipe_last_error": (ctypes.c_char_p, [P]),
        "autopipe_load_profile": (i32, [P, u32, pu64, pu64, pu64]),
        "autopipe_set_state": (i32, [P, u32, pu64, pu64, pu64, P]),
        "autopipe_set_state_device": (i32, [P, u32, P, P, P, P]),
        "autopipe_eval_partitions": (i32, [P, P, u64, P, P]),
        "autopipe_search_optimum": (i32, [P, u32, u32, u32, u64, u64, ctypes.POINTER(Result), P]),
        "autopipe_rollout_rewards": (i32, [P, P, u64, ctypes.POINTER(Partition), P, P, P]),
        "autopipe_count_candidates": (i32, [P, u32, u32, u32, pu64]),
        "autopipe_decode_index": (i32, [P, u32, u32, u32, u64, ctypes.POINTER(Partition)]),
        "autopipe_int_path": (i32, [P]),
        "autopipe_kernel_launches": (u64, [P]),
        "autopipe_set_timing": (i32, [P, i32]),
        "autopipe_set_search_options": (i32, [P, u32]),
        "autopipe_local_search": (i32, [P, P, u32, P, u32, P, P]),
        "autopipe_last_search_ms": (ctypes.c_double, [P]),
        "autopipe_neighbourhood": (i32, [P, ctypes.POINTER(Partition), P, u64, pu64, P]),
        "autopipe_neighbourhood_best": (i32, [P, ctypes.POINTER(Partition), ctypes.POINTER(Result), P]),
        "autopipe_switch_rewards": (i32, [P, P, u64, ctypes.POINTER(Partition), u64, P, P, P, P, P]),
        "autopipe_balanced_shards": (i32, [u32, u32, u32, u32, u32, u32, pu64]),
        "autopipe_balanced_shards_path": (i32, [u32, u32, u32, u32, u32, u32, u32, pu64]),
        "autopipe_set_schedule": (i32, [P, u32, u32, u32, u32]),
        "autopipe_eval_partitions_w": (i32, [P, P, u64, P, P]),
        "autopipe_rollout_rewards_w": (i32, [P, P, u64, ctypes.POINTER(PartitionW), P, P, P]),
        "autopipe_search_optimum_w": (i32, [P, u32, u32, u32, u64, u64, ctypes.POINTER(ResultW), P]),
        "autopipe_decode_index_w": (i32, [P, u32, u32, u32, u64, ctypes.POINTER(PartitionW)]),
        "autopipe_get_schedule": (i32, [P] + [ctypes.POINTER(ctypes.c_uint32)] * 4),
        "autopipe_search_optimum_async": (i32, [P, u32, u32, u32, u64, u64, P, P]),
        "autopipe_search_optimum_async_w": (i32, [P, u32, u32, u32, u64, u64, P, P]),
        "autopipe_search_seed_async": (i32, [P, u32, u32, u32, u64, u64, P, P]),
        "autopipe_set_search_bound": (i32, [P, P]),
        "autopipe_reduce_results": (i32, [P, u32, P, P]),
        "autopipe_reduce_results_w": (i32, [P, u32, P, P]),
        "autopipe_search_times": (i32, [P, ctypes.POINTER(ctypes.c_double), u32, ctypes.POINTER(u32)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name, None)
        if fn is None and os.environ.get("AUTOPIPE_LIB"):
            continue  # an older variant build named by AUTOPIPE_LIB (experiments): calls it lacks fail
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


lib = _load()
