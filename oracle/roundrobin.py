"""Oracle: PipeDream's round-robin replicas (NEXT row f4, reading F-5). Test infrastructure only.

PipeDream's partitioner picks "a partitioning of layers with the form of stages", the "number of
workers for each stage" and the "number of on-the-fly mini-batches"; a replicated
stage of PipeDream takes whole mini-batches in turn (round-robin), unlike the split replicas of
reading C-3 (DAPPLE-style), which share every mini-batch. Reading F-5
makes that schedule exact:

* mini-batch k is processed at stage s by replica k mod r_s, i.e. worker W_s[k mod r_s], whole:
  F = sum_{l in s} f[w][l], B = sum_{l in s} b[w][l] (no division by r);
* every replica runs 1F1B over its own mini-batches k_q = i + q r_s with m_s of them in flight:
  F(k_0), ..., F(k_{m-1}), B(k_0), F(k_m), B(k_1), F(k_{m+1}), ...; m_s = ceil(R_s / r_s) with
  R_s = sum_{u >= s} r_u, PipeDream's "optimal number of on-the-fly mini-batches to fill the
  pipeline" (NOAM = ceil(#workers / #replicas of the input stage) for stage 0,
  and S - s in every stage when all r = 1, as in reading C-2);
* boundary s of mini-batch k is one transfer of O[e_s] bytes (forward) on the directed link
  W_s[k mod r_s] -> W_{s+1}[k mod r_{s+1}], started when F_s(k) has finished, and one transfer of
  G[e_s + 1] bytes (backward) on W_{s+1}[k mod r_{s+1}] -> W_s[k mod r_s] after B_{s+1}(k); FIFO per
  directed link (transfers in mini-batch order); comm never occupies a worker (C-9);
* a replicated stage synchronises its gradients once per round of its replicas (every r_s
  mini-batches: ring all-reduce over W_s, or the sharded parameter server of reading F-3); nothing
  waits for it (C-4). Its chain AR(q) = max(its inputs, AR(q-1)) + d has slope d per round, so it
  contributes d / r_s per mini-batch: lambda = max(lambda_compute, max_s d_s / r_s);
* T_ns = ceil(lambda) (C-7); with every r_s = 1 this is exactly the model of ``sim``.

lambda_compute is found by simulation. The schedule's structure repeats every
Lam = lcm(r_0, ..., r_{S-1}) mini-batches. Mini-batches fall into g = gcd(r_0, ..., r_{S-1}) classes
(k mod g) that share no worker and no link, so each class is normalised on its own. Round j groups
B_s(j) and F_s(j + D_s) of every stage (D_s = min_{u <= s} m_u r_u) with the transfers they start;
the rounds of a window of Lam + D_0 + S + 2 rounds hold every event the future depends on (each
replica acts at least every r_s rounds, each link at least every lcm(r_s, r_{s+1}) rounds, a forward
transfer is consumed at most D_0 rounds after it). The first time the window, normalised per
class, repeats at the same phase (j mod Lam), the schedule is periodic: lambda_compute = max over
classes of (shift of the class) / (rounds between the repeats). ``max_cycle_ratio`` recomputes it as
the maximum cycle ratio of the explicit timed event graph of one period (an independent
formulation, tiny instances only).
"""
from __future__ import annotations

from fractions import Fraction
from math import gcd
from typing import Dict, List, Optional, Tuple

from .model import U64_MAX, Partition, allreduce_duration, ceil_div, parse_record, xfer

RING, PS = 0, 1
MAX_ROUNDS = 200_000
TIME_NS_ROUNDS = 20_000   # time_ns waits this long for the periodic regime, then takes ceil(lambda) from
                          # the event graph (Bellman-Ford on integer theta; reading R-2's fallback)


class NoPeriod(RuntimeError):
    """The round-robin schedule did not become periodic within the allowed number of rounds."""


def lcm(a: int, b: int) -> int:
    return a * b // gcd(a, b)


class RRIngredients:
    """Per-worker whole-mini-batch op durations, per-link transfer durations, sync durations."""

    def __init__(self, prof, st, part: Partition, sync: int = RING):
        from .schedules import ps_duration
        L = len(prof.O)
        self.S = part.S
        self.W = [list(ws) for ws in part.W]
        self.r = [len(ws) for ws in self.W]
        stages = part.stage_layers(L)
        self.Fd: List[Dict[int, int]] = []
        self.Bd: List[Dict[int, int]] = []
        self.sync: List[int] = []
        for s, (a, e) in enumerate(stages):
            self.Fd.append({w: sum(st.f[w][a:e + 1]) for w in self.W[s]})
            self.Bd.append({w: sum(st.b[w][a:e + 1]) for w in self.W[s]})
            if sync == PS:
                self.sync.append(ps_duration(prof.P, a, e, self.W[s], st.tau))
            else:
                self.sync.append(allreduce_duration(prof.P, a, e, self.W[s], st.tau))
        self.Of = [prof.O[stages[s][1]] for s in range(part.S - 1)]   # forward bytes of boundary s
        self.Gb = [prof.G[stages[s][1] + 1] for s in range(part.S - 1)]  # backward bytes
        self.tau = st.tau
        self.Lam = 1
        self.g = 0
        for r in self.r:
            self.Lam = lcm(self.Lam, r)
            self.g = gcd(self.g, r)
        # in flight per replica (PipeDream's NOAM per stage) and the round offsets of the forwards
        self.m = [ceil_div(sum(self.r[s:]), self.r[s]) for s in range(self.S)]
        self.D = []
        for s in range(self.S):
            d = self.m[s] * self.r[s]
            self.D.append(d if s == 0 else min(self.D[-1], d))

    def worker(self, s: int, k: int) -> int:
        return self.W[s][k % self.r[s]]

    def fwd_time(self, s: int, k: int) -> int:
        u, v = self.worker(s, k), self.worker(s + 1, k)
        return xfer(self.Of[s], self.tau[u][v])

    def bwd_time(self, s: int, k: int) -> int:
        u, v = self.worker(s + 1, k), self.worker(s, k)
        return xfer(self.Gb[s], self.tau[u][v])


def replica_op(m: int, r: int, i: int, p: int) -> Tuple[str, int]:
    """Position p of the op list of replica i (of r, m in flight): its mini-batches are k_q = i + q r;
    F(k_0..k_{m-1}), B(k_0), F(k_m), B(k_1), F(k_{m+1}), ..."""
    if p < m:
        return ("F", i + p * r)
    q, odd = divmod(p - m, 2)
    return ("B", i + q * r) if odd == 0 else ("F", i + (q + m) * r)


class RRSchedule:
    """Ready-driven execution of the round-robin schedule: every worker runs its own subsequence of
    its stage's order; an op starts when its worker is free and its input has arrived."""

    def __init__(self, ing: RRIngredients):
        self.ing = ing
        S = ing.S
        self.F: Dict[Tuple[int, int], int] = {}   # (s, k) -> end of F_s(k)
        self.B: Dict[Tuple[int, int], int] = {}
        self.fdone: Dict[Tuple[int, int], int] = {}   # (s, k) -> forward transfer of boundary s ends
        self.bdone: Dict[Tuple[int, int], int] = {}
        self.link: Dict[Tuple[str, int, int, int], int] = {}   # directed link -> free time
        self.wfree: Dict[int, int] = {w: 0 for ws in ing.W for w in ws}
        # per worker: its stage, replica index and the next global position to scan
        self.rep = {}
        for s, ws in enumerate(ing.W):
            for i, w in enumerate(ws):
                self.rep[w] = (s, i)
        self.gpos = {w: 0 for w in self.wfree}
        self.next_f = [0] * max(S - 1, 0)   # next forward transfer to start per boundary
        self.next_b = [0] * max(S - 1, 0)
        self.rounds_done = -(10**9)

    def _next_op(self, w: int) -> Tuple[str, int, int]:
        """The worker's next op (kind, mini-batch, its list position), without consuming it."""
        s, i = self.rep[w]
        p = self.gpos[w]
        kind, k = replica_op(self.ing.m[s], self.ing.r[s], i, p)
        return kind, k, p

    def round_of(self, s: int, kind: str, k: int) -> int:
        return k if kind == "B" else k - self.ing.D[s]

    def _boundaries(self) -> bool:
        ing, progress = self.ing, False
        for s in range(ing.S - 1):
            while (s, self.next_f[s]) in self.F:
                k = self.next_f[s]
                u, v = ing.worker(s, k), ing.worker(s + 1, k)
                start = max(self.F[(s, k)], self.link.get(("f", s, u, v), 0))
                end = start + ing.fwd_time(s, k)
                self.link[("f", s, u, v)] = end
                self.fdone[(s, k)] = end
                self.next_f[s] += 1
                progress = True
            while (s + 1, self.next_b[s]) in self.B:
                k = self.next_b[s]
                u, v = ing.worker(s + 1, k), ing.worker(s, k)
                start = max(self.B[(s + 1, k)], self.link.get(("b", s, u, v), 0))
                end = start + ing.bwd_time(s, k)
                self.link[("b", s, u, v)] = end
                self.bdone[(s, k)] = end
                self.next_b[s] += 1
                progress = True
        return progress

    def run_to(self, target: int) -> None:
        """Execute every op of rounds <= target (and the transfers they start)."""
        if target <= self.rounds_done:
            return
        ing = self.ing
        while True:
            progress = False
            for w in self.wfree:
                s, _ = self.rep[w]
                while True:
                    kind, k, p = self._next_op(w)
                    if self.round_of(s, kind, k) > target:
                        break
                    if kind == "F":
                        t = 0 if s == 0 else self.fdone.get((s - 1, k))
                    else:
                        t = 0 if s == ing.S - 1 else self.bdone.get((s, k))
                    if t is None:
                        break
                    start = max(self.wfree[w], t)
                    end = start + (ing.Fd[s][w] if kind == "F" else ing.Bd[s][w])
                    (self.F if kind == "F" else self.B)[(s, k)] = end
                    self.wfree[w] = end
                    self.gpos[w] = p + 1
                    progress = True
            if self._boundaries():
                progress = True
            if not progress:
                break
        for w in self.wfree:
            s, _ = self.rep[w]
            kind, k, _p = self._next_op(w)
            if self.round_of(s, kind, k) <= target:
                raise RuntimeError("round-robin schedule deadlocked")
        self.rounds_done = target

    def round_events(self, j: int) -> List[Tuple[int, int]]:
        """(class, time) of every event of round j: B_s(j), F_s(j + D_s) and their transfers."""
        ing, g, out = self.ing, self.ing.g, []
        for s in range(ing.S):
            out.append((j % g, self.B[(s, j)]))
            k = j + ing.D[s]
            out.append((k % g, self.F[(s, k)]))
        for s in range(ing.S - 1):
            k = j + ing.D[s]
            out.append((k % g, self.fdone[(s, k)]))
            out.append((j % g, self.bdone[(s, j)]))
        return out


def compute_lambda(ing: RRIngredients, max_rounds: int = MAX_ROUNDS) -> Fraction:
    """lambda_compute of the round-robin schedule (exact), by the first repeat of the per-class
    normalised window of rounds at the same phase (see the module docstring)."""
    S, g, Lam = ing.S, ing.g, ing.Lam
    if S == 1:
        # no boundary: every replica runs F, B, F, B, ... on its own mini-batches (one in every r)
        return max(Fraction(ing.Fd[0][w] + ing.Bd[0][w], ing.r[0]) for w in ing.W[0])
    sched = RRSchedule(ing)
    win = Lam + ing.D[0] + S + 2
    seen: Dict[tuple, Tuple[int, List[int]]] = {}
    hist: List[List[Tuple[int, int]]] = []
    j = 0
    while j <= max_rounds:
        sched.run_to(j + 1)
        hist.append(sched.round_events(j))
        if len(hist) > win:
            hist.pop(0)
        if len(hist) == win:
            mins = [None] * g
            for rnd in hist:
                for c, t in rnd:
                    if mins[c] is None or t < mins[c]:
                        mins[c] = t
            key = (j % Lam,) + tuple(t - mins[c] for rnd in hist for c, t in rnd)
            if key in seen:
                j0, m0 = seen[key]
                period = j - j0
                return max(Fraction(mins[c] - m0[c], period) for c in range(g))
            seen[key] = (j, mins)
        j += 1
    raise NoPeriod("round-robin schedule not periodic within %d rounds" % max_rounds)


def rr_lambda(prof, st, part: Partition, sync: int = RING, max_rounds: int = MAX_ROUNDS) -> Fraction:
    ing = RRIngredients(prof, st, part, sync)
    lam = compute_lambda(ing, max_rounds)
    for s in range(part.S):
        if ing.r[s] >= 2:
            lam = max(lam, Fraction(ing.sync[s], ing.r[s]))
    return lam


def ceil_lambda_compute(ing: RRIngredients) -> int:
    """ceil(lambda_compute) without waiting for the periodic regime: the smallest integer theta such
    that no cycle of the one-period event graph has sum(durations) - theta * Lam * sum(tokens) > 0
    (Bellman-Ford positive-cycle test, binary search on theta). Two near-equal cycle ratios can make
    the transient arbitrarily long (one C5 record needs more than 200,000 rounds); this is exact."""
    if ing.S == 1:
        lam = compute_lambda(ing)
        return ceil_div(lam.numerator, lam.denominator)
    g = event_graph(ing)
    nodes = list(g.nodes)
    pos = {v: i for i, v in enumerate(nodes)}
    dur = [g.nodes[v]["dur"] for v in nodes]
    edges = [(pos[u], pos[v], g.edges[u, v]["tokens"]) for u, v in g.edges]

    def positive_cycle(theta: int) -> bool:
        d = [0] * len(nodes)
        for _ in range(len(nodes) + 1):
            changed = False
            for (u, v, tok) in edges:
                nd = d[u] + dur[v] - theta * ing.Lam * tok
                if nd > d[v]:
                    d[v] = nd
                    changed = True
            if not changed:
                return False
        return True

    lo, hi = -1, max(1, sum(dur))
    while hi - lo > 1:
        mid = (lo + hi) // 2
        if positive_cycle(mid):
            lo = mid
        else:
            hi = mid
    return hi


def time_ns(prof, st, part: Optional[Partition], sync: int = RING) -> int:
    """T_ns = ceil(lambda); UINT64_MAX for an invalid record."""
    if part is None:
        return U64_MAX
    ing = RRIngredients(prof, st, part, sync)
    try:
        lam = compute_lambda(ing, TIME_NS_ROUNDS)
        Tc = ceil_div(lam.numerator, lam.denominator)
    except NoPeriod:
        Tc = ceil_lambda_compute(ing)
    for s in range(part.S):
        if ing.r[s] >= 2:
            Tc = max(Tc, ceil_div(ing.sync[s], ing.r[s]))
    return Tc


def score_record(prof, st, rec: bytes, sync: int = RING) -> int:
    return time_ns(prof, st, parse_record(rec, len(prof.O), len(st.f)), sync)


# ------------------------------------------------------------------------------------------------
# cross-check: the maximum cycle ratio of the explicit timed event graph of one period
# ------------------------------------------------------------------------------------------------

def event_graph(ing: RRIngredients):
    """Nodes (kind, s, p) for phase p in [0, Lam): F_s(k), B_s(k) and the transfers Tf_s(k), Tb_s(k)
    of every mini-batch k = p (mod Lam); an edge u -> v with t tokens means v(k) waits for
    u(k - t*Lam + (p_v - p_u))... i.e. for the event of the mini-batch it depends on, t periods back.
    Built from the steady-state dependencies of mini-batches k in one period far from the start."""
    import networkx as nx
    S, Lam = ing.S, ing.Lam
    K0 = (4 * S + 4) * Lam + 4 * ing.D[0]   # a period well past the warm-up
    g = nx.DiGraph()

    def nid(kind, s, k):
        return (kind, s, k % Lam)

    def dep(kind_u, s_u, k_u, kind_v, s_v, k_v):
        g.add_edge(nid(kind_u, s_u, k_u), nid(kind_v, s_v, k_v), tokens=k_v // Lam - k_u // Lam)

    for k in range(K0, K0 + Lam):
        for s in range(S):
            w = ing.worker(s, k)
            g.add_node(nid("F", s, k), dur=ing.Fd[s][w])
            g.add_node(nid("B", s, k), dur=ing.Bd[s][w])
            # worker order: the previous op of the same replica (steady state: F(k) follows
            # B(k - m r), B(k) follows F(k + (m - 1) r))
            r, m = ing.r[s], ing.m[s]
            dep("B", s, k - m * r, "F", s, k)
            dep("F", s, k + (m - 1) * r, "B", s, k)
            if s > 0:
                dep("Tf", s - 1, k, "F", s, k)
            if s < S - 1:
                dep("Tb", s, k, "B", s, k)
        for s in range(S - 1):
            g.add_node(nid("Tf", s, k), dur=ing.fwd_time(s, k))
            g.add_node(nid("Tb", s, k), dur=ing.bwd_time(s, k))
            dep("F", s, k, "Tf", s, k)
            dep("B", s + 1, k, "Tb", s, k)
            step = lcm(ing.r[s], ing.r[s + 1])   # the previous mini-batch on the same directed link
            dep("Tf", s, k - step, "Tf", s, k)
            dep("Tb", s, k - step, "Tb", s, k)
    return g


def max_cycle_ratio(prof, st, part: Partition) -> Fraction:  # noqa: D401 (tiny instances only)
    """lambda_compute as the maximum over elementary cycles of (sum of durations) / (sum of tokens),
    per mini-batch (one token = one period of Lam mini-batches)."""
    import networkx as nx
    ing = RRIngredients(prof, st, part)
    if part.S == 1:
        return compute_lambda(ing)
    g = event_graph(ing)
    best = None
    for cyc in nx.simple_cycles(g):
        dur = sum(g.nodes[v]["dur"] for v in cyc)
        tok = sum(g.edges[cyc[i], cyc[(i + 1) % len(cyc)]]["tokens"] for i in range(len(cyc)))
        if tok == 0:
            raise ValueError("zero-token cycle: the schedule would deadlock")
        r = Fraction(dur, tok * ing.Lam)
        if best is None or r > best:
            best = r
    return best
