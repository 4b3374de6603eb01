"""Multi-GPU search: split the global index space of SPEC.md §5 into one contiguous
shard per rank, search each shard on its own GPU, and combine with a (T, index) min-loc.

The only exchange is the min-loc. On GPUs (`minloc_device`) each rank's asynchronous search leaves its
40-byte result in device memory; one NCCL all-gather (40 B per rank) and one device reduction
(autopipe_reduce_results) give every rank the global (T, index) minimum, the summed evaluated count and
the winner's record, with no host round trip until the caller reads the 40 bytes. `minloc` is the
host-value form (two all_reduce(MIN) and one SUM), used by the CPU (gloo) tests and the e2e path.
Every rank holds the full, KB-sized profile and state. The shard arithmetic is exact, so the result
is the same for every world size. Rollout batches (`rollout_distributed`) split into
one contiguous slice of records per rank; the per-record outputs stay on their rank or are
all-gathered (8 bytes per record and output) into the full batch on every rank.
"""
from __future__ import annotations

from typing import Callable, List, Optional, Tuple

import torch
import torch.distributed as dist

from .engine import SearchResult, U64_MAX, reduce_results, result_from_bytes

I64_MAX = (1 << 63) - 1


def shard_bounds(total: int, rank: int, world: int) -> Tuple[int, int]:
    """Rank r of G scans [floor(r*C/G), floor((r+1)*C/G))."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad rank/world")
    return rank * total // world, (rank + 1) * total // world


def balanced_bounds(L: int, N: int, s_min: int, s_max: int, flags: int, world: int,
                    int_path: Optional[int] = None) -> List[int]:
    """world + 1 global indices splitting the space into contiguous shards of about equal device cost
    (autopipe_balanced_shards: host-only, no GPU). Equal-candidate shards leave the last rank, whose
    rows are short, up to ~1.3x slower than the first on the 96-layer space. int_path (32 or 64, the
    state's integer path as Engine.int_path reports it) selects that path's cost model
    (autopipe_balanced_shards_path)."""
    import ctypes
    from ._lib import lib
    out = (ctypes.c_uint64 * (world + 1))()
    if int_path in (32, 64):
        rc = lib.autopipe_balanced_shards_path(L, N, s_min, s_max, flags, world, int_path, out)
    else:
        rc = lib.autopipe_balanced_shards(L, N, s_min, s_max, flags, world, out)
    if rc != 0:
        raise ValueError("autopipe_balanced_shards failed (%d)" % rc)
    return [int(x) for x in out]


def minloc(T: int, idx: int, evaluated: int, group=None, device=None) -> Tuple[int, int, int]:
    """Lexicographic (T, index) minimum over ranks, and the total evaluated count.

    An empty shard reports T = index = UINT64_MAX; int64 cannot hold it, so it travels as INT64_MAX
    (every real T is < 2^59 and every index < 2^64 - 1 fits: indices of SPEC §5 spaces are < 2^35)."""
    if device is None:
        device = torch.device("cpu")
    t = torch.tensor([T if T < I64_MAX else I64_MAX], dtype=torch.int64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    tmin = int(t.item())
    i = torch.tensor([idx if (T == tmin and idx < I64_MAX) else I64_MAX], dtype=torch.int64, device=device)
    dist.all_reduce(i, op=dist.ReduceOp.MIN, group=group)
    n = torch.tensor([evaluated], dtype=torch.int64, device=device)
    dist.all_reduce(n, op=dist.ReduceOp.SUM, group=group)
    imin = int(i.item())
    if tmin == I64_MAX:
        return U64_MAX, U64_MAX, int(n.item())
    return tmin, imin, int(n.item())


def minloc_device(res: torch.Tensor, group=None, reduce_fn: Optional[Callable] = None) -> torch.Tensor:
    """Row e: all-gather the ranks' result bytes (uint8 [40] or [56] each) and reduce them on the
    device. `reduce_fn` ([world, nbytes] -> [nbytes]) defaults to autopipe_reduce_results; the CPU
    tests pass a stand-in."""
    world = dist.get_world_size(group)
    if dist.get_backend(group) == "nccl":
        gathered = torch.empty((world, res.numel()), dtype=torch.uint8, device=res.device)
        dist.all_gather_into_tensor(gathered.view(-1), res.contiguous(), group=group)
    else:  # gloo (CPU tests, test-only bench mode): exchange host copies
        g = torch.empty((world, res.numel()), dtype=torch.uint8)
        dist.all_gather(list(g.unbind(0)), res.contiguous().cpu(), group=group)
        gathered = g.to(res.device)
    return (reduce_fn or reduce_results)(gathered)


def bound_allreduce(seed: torch.Tensor, group=None) -> torch.Tensor:
    """Row e, cross-shard bound: the minimum over the ranks of one uint64 seed word (held in an 8-byte
    int64 tensor, as autopipe_search_seed_async writes it), in place. UINT64_MAX ("no seed") reads as
    -1 in int64, so it is mapped to INT64_MAX for the MIN and back; real seeds are < 2^59."""
    v = seed.view(torch.int64)
    v.masked_fill_(v == -1, (1 << 63) - 1)
    if dist.get_backend(group) == "nccl":
        dist.all_reduce(v, op=dist.ReduceOp.MIN, group=group)
    else:  # gloo: host copy
        h = v.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.MIN, group=group)
        v.copy_(h)
    v.masked_fill_(v == (1 << 63) - 1, -1)
    return seed


def search_distributed(engine, s_min: int, s_max: int, flags: int = 0, group=None,
                       shard_search: Optional[Callable[[int, int], SearchResult]] = None,
                       device=None, balanced: bool = True,
                       reduce_fn: Optional[Callable] = None) -> SearchResult:
    """Exhaustive search of the whole space across the ranks of `group`.

    By default each rank runs the engine's asynchronous search of its shard and the ranks combine with
    `minloc_device` (the winner's record travels in its 40-byte result). `shard_search(begin, end)`
    replaces the shard search with a stand-in (the CPU tests), combined by the host-value `minloc`, the
    record then decoded from the global index on every rank. `balanced` splits by estimated device
    cost (balanced_bounds) instead of equal candidate counts; the result is the same either way.
    `reduce_fn` replaces the device reduction of `minloc_device` (the CPU tests)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    if balanced:
        path = getattr(engine, "int_path", None) if hasattr(engine, "_h") else None
        b = balanced_bounds(engine.L, engine.N, s_min, s_max, flags, world, path)
        lo, hi = b[rank], b[rank + 1]
    else:
        total = engine.count_candidates(s_min, s_max, flags)
        lo, hi = shard_bounds(total, rank, world)
    if shard_search is None:
        # the engine's asynchronous shard search + the device min-loc: one host read of 40 bytes
        out = minloc_device(engine.search_optimum_async(s_min, s_max, flags, begin=lo, end=hi), group, reduce_fn)
        return result_from_bytes(out)
    r = shard_search(lo, hi)
    T, idx, n = minloc(r.time_ns, r.index, r.evaluated, group=group, device=device)
    part = engine.decode_index(s_min, s_max, flags, idx) if idx != U64_MAX else bytes([0xFF] * 16)
    return SearchResult(T, idx, n, part)


def rollout_distributed(engine, records: torch.Tensor, current: Optional[bytes] = None, group=None,
                        gather: bool = True, score: Optional[Callable] = None):
    """Row e for the RL rollout rewards: rank r of G scores the records
    [floor(r n / G), floor((r + 1) n / G)) of the batch (every rank holds the same batch, or at least
    its slice) with the engine's autopipe_rollout_rewards. gather=False returns the rank's slice
    bounds and its outputs (T_ns, switch bytes or None); gather=True all-gathers the outputs into the
    whole batch on every rank (NCCL all_gather_into_tensor of equal, padded slices; gloo: host copies)
    and returns (T_ns, switch bytes or None) for all n records. `score(slice, current)` replaces the
    engine call (the CPU tests)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    n = int(records.shape[0])
    lo, hi = shard_bounds(n, rank, world)
    if score is None:
        t, sw = engine.rollout_rewards(records[lo:hi], current)
    else:
        t, sw = score(records[lo:hi], current)
    if not gather:
        return (lo, hi), t, sw
    per = (n + world - 1) // world  # slices padded to the longest (at most one record longer)
    outs = []
    for x in (t, sw):
        if x is None:
            outs.append(None)
            continue
        pad = torch.zeros(per, dtype=torch.int64, device=x.device)
        pad[: hi - lo] = x
        if dist.get_backend(group) == "nccl":
            full = torch.empty(world * per, dtype=torch.int64, device=x.device)
            dist.all_gather_into_tensor(full, pad, group=group)
        else:  # gloo: host copies
            parts = [torch.empty(per, dtype=torch.int64) for _ in range(world)]
            dist.all_gather(parts, pad.cpu(), group=group)
            full = torch.cat(parts).to(x.device)
        # rank q's slice starts at q * per in `full`; keep its hi_q - lo_q records
        keep = [full[q * per: q * per + (shard_bounds(n, q, world)[1] - shard_bounds(n, q, world)[0])]
                for q in range(world)]
        outs.append(torch.cat(keep))
    return outs[0], outs[1]
