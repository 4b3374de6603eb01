"""Oracle: the two-worker neighbourhood of a partition.
Test infrastructure only.

"we limit the new partition solution to only change the two workers' tasks in comparison to the
old one", where a partition is "an array with size N, each element ... the
assigned layers of each worker". Reading F-1: a worker's task is its
layer set (its stage's interval, or nothing when idle); the neighbourhood of p is every valid
partition q != p whose per-worker layer-set array differs from p's in one or two entries.

This module computes it by the definition: it enumerates every valid partition of the (tiny) space
(every S, cut set and worker-to-stage map) and keeps those at distance 1 or 2. The best neighbour
is the minimum of (T_ns, record bytes) — the record's 16 bytes break ties, so the answer does not
depend on any enumeration order.
"""
from __future__ import annotations

from itertools import combinations, product
from typing import List, Optional, Tuple

from .model import Partition, encode_partition, parse_record
from .sim import time_ns


def layer_sets(p: Partition, L: int, N: int) -> Tuple[Optional[Tuple[int, int]], ...]:
    """The paper's partition array: per worker, its stage's layer interval, or None when idle."""
    out: List[Optional[Tuple[int, int]]] = [None] * N
    for s, (a, e) in enumerate(p.stage_layers(L)):
        for w in p.W[s]:
            out[w] = (a, e)
    return tuple(out)


def all_partitions(L: int, N: int):
    """Every valid partition: S in [1, min(8, N, L)], every cut set, every worker-to-stage map in
    which each stage has at least one worker (brute force; tiny L, N only)."""
    for S in range(1, min(8, N, L) + 1):
        for cuts in combinations(range(L - 1), S - 1):
            for sow in product(list(range(S)) + [None], repeat=N):
                W = [[w for w in range(N) if sow[w] == s] for s in range(S)]
                if any(not ws for ws in W):
                    continue
                yield Partition(S, list(cuts), W)


def neighbourhood(L: int, N: int, current: Partition) -> List[bytes]:
    """Records of all q with 1 <= |{w : layers_q(w) != layers_p(w)}| <= 2, sorted by record bytes."""
    base = layer_sets(current, L, N)
    out = []
    for q in all_partitions(L, N):
        d = sum(1 for a, b in zip(layer_sets(q, L, N), base) if a != b)
        if 1 <= d <= 2:
            out.append(encode_partition(q))
    return sorted(out)


def best_neighbour(prof, st, current_rec: bytes) -> Tuple[int, bytes, int]:
    """(T_ns, record) minimum over the neighbourhood (ties: smallest record bytes), and its size."""
    L, N = len(prof.O), len(st.f)
    cur = parse_record(current_rec, L, N)
    if cur is None:
        raise ValueError("invalid current partition")
    best = ((1 << 64) - 1, bytes([0xFF] * 16))  # an empty neighbourhood (one worker, one stage)
    recs = neighbourhood(L, N, cur)
    for rec in recs:
        T = time_ns(prof, st, parse_record(rec, L, N))
        if (T, rec) < best:
            best = (T, rec)
    return best[0], best[1], len(recs)
