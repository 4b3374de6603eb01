"""Oracle: brute-force search (SPEC.md §5). Test infrastructure only.

min over the enumeration of ``sim.time_ns``; the first minimum in index order wins (reading C-13).
"""
from __future__ import annotations

from typing import Optional, Tuple

from .enumerate import candidates
from .model import Partition
from .sim import time_ns


def brute_force(prof, st, s_min: int, s_max: int, flags: int = 0,
                begin: int = 0, end: Optional[int] = None) -> Tuple[int, int, Optional[Partition], int]:
    """Returns (T_ns, index, partition, evaluated) of the lexicographic minimum over [begin, end)."""
    L, N = len(prof.O), len(st.f)
    best = (None, None, None)
    n = 0
    for idx, part in enumerate(candidates(L, N, s_min, s_max, flags)):
        if idx < begin:
            continue
        if end is not None and idx >= end:
            break
        T = time_ns(prof, st, part)
        n += 1
        if best[0] is None or T < best[0]:
            best = (T, idx, part)
    return best[0], best[1], best[2], n
