"""Oracle pin for search optima: an exact parametric DP. Test infrastructure only.

Independent of ``sim`` (it works on the cycle terms of SPEC §4, not on the event schedule) and of the
GPU path (shares no code). It is itself pinned against ``search.brute_force`` on small spaces
(tests/test_oracle_dp.py), and then pins the GPU search at sizes no brute force can reach (the
96-layer, 8-stage space of 1.1e10 candidates).

For an integer theta, T <= theta iff every term of SPEC §4 is <= theta; for a segment term
ceil(W(s,t)/(t-s+1)) <= theta iff W(s,t) <= theta*(t-s+1). Scanning the stages left to right with the
"open excess" O_t = max over s <= t of [X_s - theta + sum_{s<u<=t}(Y_u - theta) + sum_{u=s}^{t-1} z_u]
(Y = Fm + Bm, z = cf + cb), every segment closing at t is checked by O_{t-1} + z_{t-1} + X_t <= theta and
O_t = max(X_t - theta, O_{t-1} + z_{t-1} + Y_t - theta). Both are monotone in O_{t-1}, so keeping the
smallest O per (stage, last layer) is exact. Binary search on theta gives the optimum; a backward pass
(largest O from which a completion exists) plus a forward greedy gives the lexicographically-first
cut set. Compositions and S are scanned in index order (SPEC §5), so the result is the global
(T, smallest index) minimum.
"""
from __future__ import annotations

from math import comb
from typing import Dict, List, Optional, Tuple

from .enumerate import USE_ALL_WORKERS, compositions, index_of
from .model import Partition, allreduce_duration, boundary_transfers, ceil_div

NEG = None  # "no feasible completion"


class _Tables:
    """X, Y, AR per (worker set, a, e) and cf, cb per (sender set, receiver set, e)."""

    def __init__(self, prof, st):
        self.prof, self.st = prof, st
        self.L = len(prof.O)
        self.pf = [[0] for _ in st.f]
        self.pb = [[0] for _ in st.b]
        for w in range(len(st.f)):
            for l in range(self.L):
                self.pf[w].append(self.pf[w][-1] + st.f[w][l])
                self.pb[w].append(self.pb[w][-1] + st.b[w][l])
        self.stage_cache: Dict[tuple, Tuple[int, int, int]] = {}
        self.bnd_cache: Dict[tuple, Tuple[int, int]] = {}

    def stage(self, ws: tuple, a: int, e: int) -> Tuple[int, int, int]:
        key = (ws, a, e)
        v = self.stage_cache.get(key)
        if v is None:
            r = len(ws)
            Fd = [ceil_div(self.pf[w][e + 1] - self.pf[w][a], r) for w in ws]
            Bd = [ceil_div(self.pb[w][e + 1] - self.pb[w][a], r) for w in ws]
            X = max(x + y for x, y in zip(Fd, Bd))
            Y = max(Fd) + max(Bd)
            AR = allreduce_duration(self.prof.P, a, e, list(ws), self.st.tau)
            v = (X, Y, AR)
            self.stage_cache[key] = v
        return v

    def boundary(self, ws: tuple, wn: tuple, e: int) -> Tuple[int, int]:
        key = (ws, wn, e)
        v = self.bnd_cache.get(key)
        if v is None:
            fw = boundary_transfers(self.prof.O[e], list(ws), list(wn), self.st.tau)
            bw = boundary_transfers(self.prof.G[e + 1], list(wn), list(ws), self.st.tau)
            v = (max([d for _, _, d in fw], default=0), max([d for _, _, d in bw], default=0))
            self.bnd_cache[key] = v
        return v


def _worker_sets(R) -> List[tuple]:
    R0 = [0] + list(R)
    return [tuple(range(R0[s], R0[s + 1])) for s in range(len(R))]


def _forward_feasible(tb: _Tables, Ws: List[tuple], theta: int) -> bool:
    L, S = tb.L, len(Ws)
    # best[e] = smallest open excess with the current stage ending at layer e
    best: Dict[int, int] = {}
    for e in range(0, L - S + 1):
        X, Y, AR = tb.stage(Ws[0], 0, e)
        if X <= theta and AR <= theta:
            best[e] = X - theta
    for t in range(1, S):
        nxt: Dict[int, int] = {}
        e_hi = L - 1 if t == S - 1 else L - S + t
        for ep, O in best.items():
            cf, cb = tb.boundary(Ws[t - 1], Ws[t], ep)
            if cf > theta or cb > theta:
                continue
            z = cf + cb
            for e in (range(ep + 1, e_hi + 1) if t < S - 1 else [L - 1]):
                if e <= ep:
                    continue
                X, Y, AR = tb.stage(Ws[t], ep + 1, e)
                if X > theta or AR > theta or O + z + X - theta > 0:
                    continue
                On = max(X - theta, O + z + Y - theta)
                if e not in nxt or On < nxt[e]:
                    nxt[e] = On
        best = nxt
        if not best:
            return False
    return (L - 1) in best


def _lex_first_cuts(tb: _Tables, Ws: List[tuple], theta: int) -> Optional[List[int]]:
    L, S = tb.L, len(Ws)
    INF = 1 << 200
    # Omax[t][e]: largest O_t at (stage t ends at e) from which the remaining stages are feasible
    Omax: List[Dict[int, int]] = [dict() for _ in range(S)]
    Omax[S - 1][L - 1] = INF
    for t in range(S - 2, -1, -1):
        for e in range(t, L - 1 - (S - 2 - t)):
            cf, cb = tb.boundary(Ws[t], Ws[t + 1], e)
            if cf > theta or cb > theta:
                continue
            z = cf + cb
            bestO = NEG
            for en, Onext in Omax[t + 1].items():
                if en <= e:
                    continue
                X, Y, AR = tb.stage(Ws[t + 1], e + 1, en)
                if X > theta or AR > theta or X - theta > Onext:
                    continue
                bound = min(theta - z - X, Onext - z - Y + theta)
                if bestO is NEG or bound > bestO:
                    bestO = bound
            if bestO is not NEG:
                Omax[t][e] = bestO
    cuts: List[int] = []
    if S == 1:
        X, Y, AR = tb.stage(Ws[0], 0, L - 1)
        return [] if (X <= theta and AR <= theta) else None
    O, ep = None, None
    for t in range(0, S - 1):
        chosen = None
        lo = 0 if t == 0 else ep + 1
        for e in range(lo, L - 1 - (S - 2 - t)):
            if e not in Omax[t]:
                continue
            X, Y, AR = tb.stage(Ws[t], lo, e)
            if X > theta or AR > theta:
                continue
            if t == 0:
                On = X - theta
            else:
                cf, cb = tb.boundary(Ws[t - 1], Ws[t], ep)
                z = cf + cb
                if cf > theta or cb > theta or O + z + X - theta > 0:
                    continue
                On = max(X - theta, O + z + Y - theta)
            if On <= Omax[t][e]:
                chosen = (e, On)
                break
        if chosen is None:
            return None
        ep, O = chosen
        cuts.append(ep)
    return cuts


def optimum(prof, st, s_min: int, s_max: int, flags: int = 0, hi: Optional[int] = None
            ) -> Tuple[int, int, Partition]:
    """Exact search optimum: (T_ns, global index of the lexicographically-first argmin, partition)."""
    tb = _Tables(prof, st)
    L, N = tb.L, len(st.f)
    structs = []
    for S in range(s_min, s_max + 1):
        if S > L:
            continue
        for R in compositions(N, S, flags):
            structs.append((S, _worker_sets(R)))
    if not structs:
        raise ValueError("empty search space")

    def feasible(theta):
        return any(_forward_feasible(tb, Ws, theta) for _, Ws in structs)

    if hi is None:
        hi = 1
        while not feasible(hi):
            hi *= 2
    lo = -1                       # infeasible (T >= 0 always)
    while hi - lo > 1:
        mid = (lo + hi) // 2
        if feasible(mid):
            hi = mid
        else:
            lo = mid
    theta = hi
    for S, Ws in structs:
        if _forward_feasible(tb, Ws, theta):
            cuts = _lex_first_cuts(tb, Ws, theta)
            part = Partition(S, cuts, [list(w) for w in Ws])
            return theta, index_of(L, N, s_min, s_max, flags, part), part
    raise AssertionError("unreachable")
