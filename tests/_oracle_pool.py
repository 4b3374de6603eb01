"""Parallel evaluation of the oracle over many records (test infrastructure)."""
from __future__ import annotations

import multiprocessing as mp
import os
from typing import List, Sequence

_CTX = {}


def _init(prof, st):
    _CTX["prof"] = prof
    _CTX["st"] = st


def _score(rec: bytes) -> int:
    from oracle.sim import score_record
    return score_record(_CTX["prof"], _CTX["st"], rec)


def _score_pair(args):
    from oracle.rollout import rollout_rewards
    rec, cur = args
    t, sw = rollout_rewards(_CTX["prof"], _CTX["st"], [rec], cur)
    return t[0], (sw[0] if sw is not None else None)


def cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def score_many(prof, st, records: Sequence[bytes], procs: int = 0) -> List[int]:
    records = [bytes(r) for r in records]
    procs = procs or cores()
    if procs <= 1 or len(records) < 64:
        _init(prof, st)
        return [_score(r) for r in records]
    with mp.get_context("fork").Pool(procs, initializer=_init, initargs=(prof, st)) as pool:
        return pool.map(_score, records, chunksize=max(1, len(records) // (procs * 8)))


def rollout_many(prof, st, records: Sequence[bytes], current, procs: int = 0):
    records = [bytes(r) for r in records]
    procs = procs or cores()
    args = [(r, current) for r in records]
    if procs <= 1 or len(records) < 64:
        _init(prof, st)
        out = [_score_pair(a) for a in args]
    else:
        with mp.get_context("fork").Pool(procs, initializer=_init, initargs=(prof, st)) as pool:
            out = pool.map(_score_pair, args, chunksize=max(1, len(args) // (procs * 8)))
    return [o[0] for o in out], [o[1] for o in out]


def _switch_one(args):
    from oracle.model import parse_record
    from oracle.switching import switch_reward
    rec, cur, horizon = args
    p = parse_record(cur, len(_CTX["prof"].O), len(_CTX["st"].f))
    return switch_reward(_CTX["prof"], _CTX["st"], rec, p, horizon)


def switch_many(prof, st, records: Sequence[bytes], current: bytes, horizon: int, procs: int = 0):
    """oracle.switching.switch_reward over many proposals: list of (T, refill, migrate, reward)."""
    args = [(bytes(r), bytes(current), horizon) for r in records]
    procs = procs or cores()
    if procs <= 1 or len(args) < 64:
        _init(prof, st)
        return [_switch_one(a) for a in args]
    with mp.get_context("fork").Pool(procs, initializer=_init, initargs=(prof, st)) as pool:
        return pool.map(_switch_one, args, chunksize=max(1, len(args) // (procs * 8)))


def _sched_one(args):
    from oracle.schedules import score_record
    rec, model = args
    return score_record(_CTX["prof"], _CTX["st"], rec, *model)


def sched_many(prof, st, records: Sequence[bytes], schedule: int, sync: int, M: int, recompute: bool,
               procs: int = 0) -> List[int]:
    """oracle.schedules.score_record (row f3) over many records."""
    model = (schedule, sync, M, recompute)
    args = [(bytes(r), model) for r in records]
    procs = procs or cores()
    if procs <= 1 or len(args) < 64:
        _init(prof, st)
        return [_sched_one(a) for a in args]
    with mp.get_context("fork").Pool(procs, initializer=_init, initargs=(prof, st)) as pool:
        return pool.map(_sched_one, args, chunksize=max(1, len(args) // (procs * 8)))


def _rr_one(args):
    from oracle.roundrobin import score_record
    rec, sync = args
    return score_record(_CTX["prof"], _CTX["st"], rec, sync)


def rr_many(prof, st, records: Sequence[bytes], sync: int = 0, procs: int = 0) -> List[int]:
    """oracle.roundrobin.score_record (row f4, round-robin replicas) over many records."""
    args = [(bytes(r), sync) for r in records]
    procs = procs or cores()
    if procs <= 1 or len(args) < 64:
        _init(prof, st)
        return [_rr_one(a) for a in args]
    with mp.get_context("fork").Pool(procs, initializer=_init, initargs=(prof, st)) as pool:
        return pool.map(_rr_one, args, chunksize=max(1, len(args) // (procs * 8)))


def _ch_one(args):
    from oracle.chimera import score_record
    rec, M, sync = args
    return score_record(_CTX["prof"], _CTX["st"], rec, M, sync)


def chimera_many(prof, st, records: Sequence[bytes], M: int, sync: int = 0, procs: int = 0) -> List[int]:
    """oracle.chimera.score_record (row f3, Chimera) over many records."""
    args = [(bytes(r), M, sync) for r in records]
    procs = procs or cores()
    if procs <= 1 or len(args) < 64:
        _init(prof, st)
        return [_ch_one(a) for a in args]
    with mp.get_context("fork").Pool(procs, initializer=_init, initargs=(prof, st)) as pool:
        return pool.map(_ch_one, args, chunksize=max(1, len(args) // (procs * 8)))
