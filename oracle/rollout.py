"""Oracle: RL rollout rewards (SPEC.md §6). Test infrastructure only.

The arbiter's input is the environment metrics, the current partition and the new one
(PAPER.md:918-921); its reward is the one-iteration training speed with a normalised switching cost
(PAPER.md:924-927). Per proposal this returns T_ns (``sim``) and the switch bytes of SPEC §6.
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

from .model import U64_MAX, parse_record, switch_bytes
from .sim import time_ns


def rollout_rewards(prof, st, records: Sequence[bytes], current: Optional[bytes]
                    ) -> Tuple[List[int], Optional[List[int]]]:
    L, N = len(prof.O), len(st.f)
    cur = parse_record(current, L, N) if current is not None else None
    if current is not None and cur is None:
        raise ValueError("invalid current partition")  # the C-ABI returns AUTOPIPE_E_INVAL
    times, sw = [], ([] if current is not None else None)
    for rec in records:
        p = parse_record(rec, L, N)
        times.append(time_ns(prof, st, p))
        if sw is not None:
            sw.append(U64_MAX if p is None else switch_bytes(prof, p, cur))
    return times, sw
