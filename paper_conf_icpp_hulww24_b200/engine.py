"""Python API over the C-ABI (include/autopipe.h): argument marshalling only.

Every score is computed by the sm_100a kernels of ``libautopipe.so``; torch is used for device
memory and streams. Outputs that the C-ABI defines as ``uint64`` come back as ``torch.int64`` tensors
holding the same bits (UINT64_MAX reads as -1); ``as_u64`` converts them to numpy uint64.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass
from typing import Optional, Sequence, Tuple

import numpy as np
import torch

from . import _lib
from ._lib import AutopipeError, Partition, PartitionW, Result, ResultW, USE_ALL_WORKERS, lib

U64_MAX = (1 << 64) - 1


def _u64_array(x, n: Optional[int] = None) -> np.ndarray:
    a = np.ascontiguousarray(np.asarray(x, dtype=np.uint64).reshape(-1))
    if n is not None and a.size != n:
        raise ValueError("expected %d values, got %d" % (n, a.size))
    return a


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))


def as_u64(t: torch.Tensor) -> np.ndarray:
    """Reinterpret an int64 tensor written by the kernels as uint64 (host copy)."""
    return t.detach().cpu().numpy().view(np.uint64)


def record_bytes(p: Partition) -> bytes:
    return bytes(bytearray(p))


@dataclass
class SearchResult:
    time_ns: int
    index: int
    evaluated: int
    partition: bytes   # the 16-byte record of the best candidate

    @property
    def empty(self) -> bool:
        return self.index == U64_MAX


def result_from_bytes(b) -> SearchResult:
    """A SearchResult from the bytes of an autopipe_result (40) or autopipe_result_w (56)."""
    raw = bytes(b.cpu().numpy().tobytes()) if isinstance(b, torch.Tensor) else bytes(b)
    if len(raw) not in (40, 56):
        raise ValueError("an autopipe_result is 40 or 56 bytes, got %d" % len(raw))
    t, i, n = (int.from_bytes(raw[k:k + 8], "little") for k in (0, 8, 16))
    return SearchResult(t, i, n, raw[24:])


def reduce_results(gathered: torch.Tensor, stream=None) -> torch.Tensor:
    """Row e: device uint8 [n, 40] (or [n, 56]) results -> [40] (or [56]): the lexicographic
    (time_ns, index) minimum, evaluated summed, the winner's record (autopipe_reduce_results)."""
    if gathered.dim() != 2 or gathered.shape[1] not in (40, 56) or gathered.dtype != torch.uint8 \
            or not gathered.is_cuda or not gathered.is_contiguous():
        raise ValueError("gathered must be a contiguous CUDA uint8 tensor [n, 40] or [n, 56]")
    out = torch.empty(gathered.shape[1], dtype=torch.uint8, device=gathered.device)
    fn = lib.autopipe_reduce_results_w if gathered.shape[1] == 56 else lib.autopipe_reduce_results
    if stream is None:
        stream = torch.cuda.current_stream(gathered.device)
    with torch.cuda.device(gathered.device):
        rc = fn(ctypes.c_void_p(gathered.data_ptr()), gathered.shape[0], ctypes.c_void_p(out.data_ptr()),
                ctypes.c_void_p(stream.cuda_stream))
    if rc != 0:
        raise AutopipeError(rc, "autopipe_reduce_results")
    return out


class Engine:
    """One engine per CUDA device (not thread-safe), mirroring ``autopipe_ctx``."""

    def __init__(self, device: int = 0):
        if not torch.cuda.is_available():
            raise RuntimeError("the AutoPipe cost-model engine needs a CUDA device (no CPU fallback)")
        self.device = torch.device("cuda", device)
        h = ctypes.c_void_p()
        rc = lib.autopipe_create(int(device), ctypes.byref(h))
        if rc != 0:
            raise AutopipeError(rc, lib.autopipe_last_error(None).decode())
        self._h = h
        self.L = 0
        self.N = 0

    def close(self):
        if getattr(self, "_h", None):
            lib.autopipe_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc: int):
        if rc != 0:
            raise AutopipeError(rc, lib.autopipe_last_error(self._h).decode())

    def _stream(self, stream=None):
        s = stream if stream is not None else torch.cuda.current_stream(self.device)
        return ctypes.c_void_p(s.cuda_stream)

    # -- Table 1 inputs --------------------------------------------------------------------
    def load_profile(self, O: Sequence[int], G: Sequence[int], P: Sequence[int]) -> None:
        o, g, p = _u64_array(O), _u64_array(G), _u64_array(P)
        if not (o.size == g.size == p.size):
            raise ValueError("O, G, P must have the same length L")
        self._check(lib.autopipe_load_profile(self._h, o.size, _ptr(o), _ptr(g), _ptr(p)))
        self.L = int(o.size)

    def set_state(self, fp, bp, tau, stream=None) -> None:
        f = np.asarray(fp, dtype=np.uint64)
        N = int(f.shape[0]) if f.ndim == 2 else len(fp)
        fa = _u64_array(fp, N * self.L)
        ba = _u64_array(bp, N * self.L)
        ta = _u64_array(tau, N * N)
        self._check(lib.autopipe_set_state(self._h, N, _ptr(fa), _ptr(ba), _ptr(ta), self._stream(stream)))
        self.N = N

    def set_state_device(self, fp: torch.Tensor, bp: torch.Tensor, tau: torch.Tensor, stream=None) -> None:
        """State from device tensors (int64/uint64 bits, shapes [N, L], [N, L], [N, N]); no host copy."""
        for t in (fp, bp, tau):
            if t.device != self.device or t.dtype not in (torch.int64, torch.uint64) or not t.is_contiguous():
                raise ValueError("state tensors must be contiguous 64-bit tensors on the engine's device")
        N = int(fp.shape[0])
        if fp.numel() != N * self.L or bp.numel() != N * self.L or tau.numel() != N * N:
            raise ValueError("expected fp, bp of shape [N, L] and tau of shape [N, N]")
        self._check(lib.autopipe_set_state_device(self._h, N, ctypes.c_void_p(fp.data_ptr()),
                                                  ctypes.c_void_p(bp.data_ptr()),
                                                  ctypes.c_void_p(tau.data_ptr()), self._stream(stream)))
        self.N = N

    def load(self, profile, state, stream=None) -> None:
        """Convenience: load_profile + set_state from workloads.Profile / workloads.State objects."""
        self.load_profile(profile.O, profile.G, profile.P)
        self.set_state(state.f, state.b, state.tau, stream)

    # -- scoring ---------------------------------------------------------------------------
    def _records(self, parts) -> torch.Tensor:
        """Records as a contiguous uint8 device tensor [n, 16] (or [n, 32]: wide records, row f4)."""
        if not isinstance(parts, torch.Tensor):
            a = np.asarray(parts, dtype=np.uint8)
            width = a.shape[-1] if a.ndim == 2 else 16
            parts = torch.as_tensor(a.reshape(-1, width))
        if parts.dtype != torch.uint8 or parts.dim() != 2 or parts.shape[1] not in (16, 32):
            raise ValueError("partitions must be a uint8 tensor of shape [n, 16] or [n, 32]")
        if parts.device != self.device:
            parts = parts.to(self.device)
        return parts.contiguous()

    def eval_partitions(self, parts, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
        recs = self._records(parts)
        n = recs.shape[0]
        if out is None:
            out = torch.empty(n, dtype=torch.int64, device=self.device)
        fn = lib.autopipe_eval_partitions_w if recs.shape[1] == 32 else lib.autopipe_eval_partitions
        self._check(fn(self._h, ctypes.c_void_p(recs.data_ptr()), n, ctypes.c_void_p(out.data_ptr()),
                       self._stream(stream)))
        return out

    def rollout_rewards(self, parts, current: Optional[bytes] = None, out_t=None, out_sw=None,
                        stream=None) -> Tuple[torch.Tensor, Optional[torch.Tensor]]:
        recs = self._records(parts)
        n = recs.shape[0]
        wide = recs.shape[1] == 32
        if out_t is None:
            out_t = torch.empty(n, dtype=torch.int64, device=self.device)
        cur = None
        if current is not None:
            cur = (PartitionW if wide else Partition).from_buffer_copy(bytes(current))
            if out_sw is None:
                out_sw = torch.empty(n, dtype=torch.int64, device=self.device)
        else:
            out_sw = None
        self._check((lib.autopipe_rollout_rewards_w if wide else lib.autopipe_rollout_rewards)(
            self._h, ctypes.c_void_p(recs.data_ptr()), n, ctypes.byref(cur) if cur is not None else None,
            ctypes.c_void_p(out_t.data_ptr()),
            ctypes.c_void_p(out_sw.data_ptr()) if out_sw is not None else None, self._stream(stream)))
        return out_t, out_sw

    def switch_rewards(self, parts, current: bytes, horizon: int, outputs=("time", "refill", "migrate"),
                       stream=None) -> dict:
        """NEXT row f2 (reading F-2): per proposal, the reward
        T_ns + ceil((refill_ns + migrate_ns) / horizon) versus the current partition. Returns a dict
        of int64 tensors: "reward" always, plus each name in `outputs`."""
        recs = self._records(parts)
        n = recs.shape[0]
        cur = Partition.from_buffer_copy(bytes(current))
        out = {k: torch.empty(n, dtype=torch.int64, device=self.device)
               for k in ("reward",) + tuple(outputs)}

        def ptr(k):
            return ctypes.c_void_p(out[k].data_ptr()) if k in out else None
        self._check(lib.autopipe_switch_rewards(
            self._h, ctypes.c_void_p(recs.data_ptr()), n, ctypes.byref(cur), int(horizon), ptr("time"),
            ptr("refill"), ptr("migrate"), ptr("reward"), self._stream(stream)))
        return out

    def _wide(self, s_max: int, wide: Optional[bool]) -> bool:
        """Spaces with S > 8 or N > 8 workers need 32-byte records (row f4)."""
        return (s_max > 8 or self.N > 8) if wide is None else bool(wide)

    def search_optimum(self, s_min: int, s_max: int, flags: int = 0, begin: int = 0,
                       end: Optional[int] = None, stream=None, wide: Optional[bool] = None) -> SearchResult:
        """Exhaustive search of [begin, end) of the space; the result's partition is a 16-byte record,
        or a 32-byte one for a wide space (S > 8 or N > 8, or wide=True)."""
        w = self._wide(s_max, wide)
        res = ResultW() if w else Result()
        e = U64_MAX if end is None else int(end)
        fn = lib.autopipe_search_optimum_w if w else lib.autopipe_search_optimum
        self._check(fn(self._h, s_min, s_max, flags, int(begin), e, ctypes.byref(res), self._stream(stream)))
        return SearchResult(int(res.time_ns), int(res.index), int(res.evaluated), record_bytes(res.part))

    def search_optimum_async(self, s_min: int, s_max: int, flags: int = 0, begin: int = 0,
                             end: Optional[int] = None, out: Optional[torch.Tensor] = None, stream=None,
                             wide: Optional[bool] = None) -> torch.Tensor:
        """The same search, enqueued on the stream with no host wait: the result is a device uint8
        tensor of 40 bytes (56 for a wide space) in the autopipe_result layout (decode a host copy
        with `result_from_bytes`). A state set from device memory is not read back (both integer
        paths are enqueued, the state kernel's choice gates them)."""
        w = self._wide(s_max, wide)
        nb = 56 if w else 40
        if out is None:
            out = torch.empty(nb, dtype=torch.uint8, device=self.device)
        if out.numel() != nb or out.dtype != torch.uint8 or out.device != self.device or not out.is_contiguous():
            raise ValueError("out must be a contiguous uint8 tensor of %d bytes on %s" % (nb, self.device))
        e = U64_MAX if end is None else int(end)
        fn = lib.autopipe_search_optimum_async_w if w else lib.autopipe_search_optimum_async
        self._check(fn(self._h, s_min, s_max, flags, int(begin), e, ctypes.c_void_p(out.data_ptr()),
                       self._stream(stream)))
        return out

    # -- row e: the cross-shard bound (autopipe_search_seed_async / autopipe_set_search_bound) --
    def search_seed_async(self, s_min: int, s_max: int, flags: int = 0, begin: int = 0,
                          end: Optional[int] = None, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
        """The shard's seed T (exact T of one of its candidates) as a device int64 [1] tensor holding a
        uint64 (UINT64_MAX when no r = 1 block of the shard is seeded); min-reduce it over the ranks
        and pass it to `set_search_bound`."""
        if out is None:
            out = torch.empty(1, dtype=torch.int64, device=self.device)
        if out.numel() != 1 or out.element_size() != 8 or out.device != self.device:
            raise ValueError("out must be one 8-byte element on %s" % self.device)
        e = U64_MAX if end is None else int(end)
        self._check(lib.autopipe_search_seed_async(self._h, s_min, s_max, flags, int(begin), e,
                                                   ctypes.c_void_p(out.data_ptr()), self._stream(stream)))
        return out

    def set_search_bound(self, bound: Optional[torch.Tensor]) -> None:
        """Later searches start their r = 1 sweeps from the device word `bound` (None clears it); the
        tensor is kept alive while it is set."""
        if bound is not None and (bound.device != self.device or bound.element_size() != 8):
            raise ValueError("bound must be one 8-byte element on %s" % self.device)
        self._bound = bound
        self._check(lib.autopipe_set_search_bound(self._h, ctypes.c_void_p(bound.data_ptr() if bound is not None else 0)))

    # -- NEXT row f1: the two-worker neighbourhood ------------------------
    def neighbourhood(self, current: bytes, capacity: int = 1 << 15, stream=None) -> torch.Tensor:
        """All partitions differing from `current` in one or two workers' layer sets (uint8 [n, 16])."""
        cur = Partition.from_buffer_copy(bytes(current))
        out = torch.empty((capacity, 16), dtype=torch.uint8, device=self.device)
        n = ctypes.c_uint64()
        self._check(lib.autopipe_neighbourhood(self._h, ctypes.byref(cur), ctypes.c_void_p(out.data_ptr()),
                                               capacity, ctypes.byref(n), self._stream(stream)))
        if n.value > capacity:
            return self.neighbourhood(current, int(n.value), stream)
        return out[: n.value]

    def best_neighbour(self, current: bytes, stream=None) -> SearchResult:
        """The neighbour with the smallest (T_ns, record bytes); evaluated = neighbourhood size."""
        cur = Partition.from_buffer_copy(bytes(current))
        res = Result()
        self._check(lib.autopipe_neighbourhood_best(self._h, ctypes.byref(cur), ctypes.byref(res),
                                                    self._stream(stream)))
        return SearchResult(int(res.time_ns), int(res.index), int(res.evaluated), record_bytes(res.part))

    def local_search(self, start: bytes, max_steps: int = 100):
        """The paper's gradual migration (autopipe_local_search): move to the best
        two-worker neighbour while it is strictly faster. Returns the path [(T_ns, record), ...]
        starting at `start`."""
        cap = max_steps + 1
        path = (Result * cap)()
        n = ctypes.c_uint32()
        cur = Partition.from_buffer_copy(bytes(start))
        self._check(lib.autopipe_local_search(self._h, ctypes.byref(cur), int(max_steps), path, cap,
                                              ctypes.byref(n), self._stream()))
        return [(int(path[i].time_ns), record_bytes(path[i].part)) for i in range(n.value)]

    # -- NEXT row f3: schedule variants (reading F-3) -----
    def set_schedule(self, schedule: int = _lib.SCHED_PIPEDREAM, sync: int = _lib.SYNC_RING,
                     micro_batches: int = 1, recompute: bool = False) -> None:
        """Select the model every later scoring call evaluates: the schedule (SCHED_PIPEDREAM, _2BW,
        _GPIPE, _DAPPLE, or SCHED_PIPEDREAM_RR: round-robin replicas, row f4), the data-parallel sync
        (SYNC_RING, SYNC_PS), M micro-batches per iteration and GPipe's forward recomputation. Times
        are then per iteration of M micro-batches."""
        self._check(lib.autopipe_set_schedule(self._h, int(schedule), int(sync), int(micro_batches),
                                              _lib.RECOMPUTE if recompute else 0))

    def get_schedule(self) -> Tuple[int, int, int, bool]:
        v = [ctypes.c_uint32() for _ in range(4)]
        self._check(lib.autopipe_get_schedule(self._h, *[ctypes.byref(x) for x in v]))
        return v[0].value, v[1].value, v[2].value, bool(v[3].value & _lib.RECOMPUTE)

    # -- support ---------------------------------------------------------------------------
    def count_candidates(self, s_min: int, s_max: int, flags: int = 0) -> int:
        v = ctypes.c_uint64()
        self._check(lib.autopipe_count_candidates(self._h, s_min, s_max, flags, ctypes.byref(v)))
        return int(v.value)

    def decode_index(self, s_min: int, s_max: int, flags: int, index: int, wide: Optional[bool] = None) -> bytes:
        w = self._wide(s_max, wide)
        p = PartitionW() if w else Partition()
        fn = lib.autopipe_decode_index_w if w else lib.autopipe_decode_index
        self._check(fn(self._h, s_min, s_max, flags, int(index), ctypes.byref(p)))
        return record_bytes(p)

    @property
    def int_path(self) -> int:
        return int(lib.autopipe_int_path(self._h))

    def set_search_options(self, split: bool = False, no_r1: bool = False, rr_defer_all: bool = False,
                           rr_no_defer: bool = False) -> None:
        """Kernel selection of later calls (autopipe_set_search_options; never changes a result):
        split=True always uses the per-S split (r = 1 sweep + threshold walk), even for ranges the dense
        launch would take; no_r1=True sends the r = 1 blocks through the threshold walk too;
        rr_defer_all / rr_no_defer: round-robin evaluations defer (nearly) every record to the
        warp-per-record drain kernel / none."""
        self._check(lib.autopipe_set_search_options(
            self._h, (1 if split else 0) | (2 if no_r1 else 0) | (4 if rr_defer_all else 0) | (8 if rr_no_defer else 0)))

    def set_timing(self, enable: bool = True) -> None:
        self._check(lib.autopipe_set_timing(self._h, 1 if enable else 0))

    @property
    def last_search_ms(self) -> float:
        """Device time of the enumeration kernels of the last search (needs set_timing(True))."""
        return float(lib.autopipe_last_search_ms(self._h))

    def search_times(self) -> list:
        """Enumeration-kernel times (ms) of the timed searches since the previous call, oldest first
        (the last 64 at most; waits for them)."""
        buf = (ctypes.c_double * 64)()
        n = ctypes.c_uint32()
        self._check(lib.autopipe_search_times(self._h, buf, 64, ctypes.byref(n)))
        return [float(buf[i]) for i in range(n.value)]

    @property
    def kernel_launches(self) -> int:
        return int(lib.autopipe_kernel_launches(self._h))
