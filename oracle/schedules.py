"""Oracle: schedule variants and parameter-server synchronisation (NEXT row f3). Test infrastructure only.

The paper sets PipeDream's asynchronous 1F1B pipeline against the
synchronous pipelines that flush — GPipe, "each mini-batch is divided into multiple smaller
micro-batches", recomputing the forward pass, and DAPPLE — and
against PipeDream-2BW's double-buffered weights with "weight gradient coalescing";
it applies AutoPipe to DAPPLE, Chimera and 2BW and synchronises the
data-parallel part with either a parameter server (PS) or ring all-reduce (PAPER.md:1081-1082,
1114-1117). DESIGN.md reading F-3 turns these into exact integer models; this module computes them
by their definitions:

* the profile (FP, BP, O, G) describes one micro-batch — the unit a stage processes; an iteration is
  M micro-batches and one weight update; every result is the time of one iteration in ns
  (PipeDream: M = 1, i.e. the existing steady-state time per mini-batch);
* PIPEDREAM  the static 1F1B steady state of ``sim`` (unchanged), replicated stages synchronised
             every mini-batch;
* TWO_BW     the same 1F1B steady state; each replicated stage synchronises once per M micro-batches
             (its chain is fed by the last micro-batch of the iteration, nothing waits for it);
             T = ceil(lambda per iteration);
* GPIPE      one iteration from an empty pipeline: every worker runs F(0..M-1), then B(0..M-1); with
             ``recompute`` each backward op first re-runs the forward (duration F' + B');
* DAPPLE     one iteration from an empty pipeline in 1F1B order: n_s = min(S - s, M) forwards, then
             B(j), F(j + n_s) while j + n_s < M, then the remaining backwards;
  for GPIPE and DAPPLE the synchronisation of a replicated stage starts when its last backward has
  finished on every replica, and T = the time the last stage finishes (its backward or its sync);
* RING  the ring all-reduce of ``model.allreduce_duration``;
* PS    a parameter server sharded over the stage's replicas: replica i serves shard i of the
        stage's weight bytes ([floor(iP/r), floor((i+1)P/r))), every other replica pushes its
        gradient of that shard to it and pulls the updated shard back; a server handles its
        incoming pushes one after another (likewise its outgoing pulls), different servers in
        parallel; PS_s = push + pull, push = max over servers v of sum over u != v of
        xfer(|shard_v|, tau[u][v]), pull = max over v of sum over u != v of xfer(|shard_v|, tau[v][u]).

Execution follows the same rules as ``sim`` (a worker runs its op list in order, an op starts when
its worker is free and its input has arrived, a boundary is a barrier over the sending replicas
followed by FIFO transfers on directed links). ``flush_makespan`` is a generic ready-driven
execution of the finite op lists; ``flush_makespan_dag`` recomputes it as the longest path of the
explicit event DAG (an independent formulation used as a cross-check on tiny instances).
"""
from __future__ import annotations

from fractions import Fraction
from math import gcd
from typing import Dict, List, Optional, Sequence, Tuple

from .model import U64_MAX, Ingredients, Partition, ceil_div, ingredients, parse_record, shards, xfer
from .sim import MAX_ROUNDS, TIME_NS_ROUNDS, NoPeriod, Schedule, steady_state, time_ns

PIPEDREAM, TWO_BW, GPIPE, DAPPLE = 0, 1, 2, 3
RING, PS = 0, 1
SCHEDULES = (PIPEDREAM, TWO_BW, GPIPE, DAPPLE)


def ps_duration(P: Sequence[int], a: int, e: int, ws: Sequence[int], tau) -> int:
    """Sharded parameter server of a replicated stage (reading F-3; PS scheme)."""
    r = len(ws)
    if r < 2:
        return 0
    sh = shards(sum(P[a:e + 1]), r)
    push = max(sum(xfer(hi - lo, tau[u][v]) for u in ws if u != v) for v, (lo, hi) in zip(ws, sh))
    pull = max(sum(xfer(hi - lo, tau[v][u]) for u in ws if u != v) for v, (lo, hi) in zip(ws, sh))
    return push + pull


def model_ingredients(prof, st, part: Partition, sync: int) -> Ingredients:
    """The ingredients of SPEC §2-3 with the stage synchronisation of ``sync`` in ``ar``."""
    ing = ingredients(prof, st, part)
    if sync == PS:
        L = len(prof.O)
        ing.ar = [ps_duration(prof.P, a, e, part.W[s], st.tau)
                  for s, (a, e) in enumerate(part.stage_layers(L))]
    return ing


# --- TWO_BW: the 1F1B steady state with one synchronisation per M micro-batches ----------------
def _coalesced_chain_slope(sched: Schedule, s: int, M: int, d: int, j0: int, c: int, D: int,
                           max_rounds: int = MAX_ROUNDS) -> Fraction:
    """Asymptotic time per iteration of the synchronisation chain of stage s when it runs once per
    M micro-batches: SY(k) = max(Bmax(kM + M - 1), SY(k-1)) + d. With o(k) = SY(k) - Bmax(kM+M-1) - d
    >= 0 and the compute events periodic from round j0 (period c rounds, shift D), k -> k + c'
    (c' = c / gcd(c, M) iterations = a whole number of compute periods) is a monotone map of o, so as
    in sim._allreduce_slope either o repeats (slope = M * D / c) or the backlog stays positive over a
    whole period and grows (slope = d)."""
    W = sched.ing.W[s]
    cp = c // gcd(c, M)
    sy: Dict[int, int] = {}

    def bmax(k: int) -> int:
        j = k * M + M - 1
        sched.ensure(j + 1)
        return max(sched.B[(s, w, j)] for w in W)

    def SY(k: int) -> int:
        for i in range(len(sy), k + 1):
            sy[i] = max(bmax(i), sy[i - 1] if i > 0 else 0) + d
        return sy[k]

    def o(k: int) -> int:
        return SY(k) - bmax(k) - d

    k = ceil_div(max(j0 - (M - 1), 0), M)
    while True:
        if o(k + cp) == o(k):
            return Fraction(M * D, c)
        if all(o(i) > 0 for i in range(k + 1, k + cp + 1)) and o(k + cp) > o(k):
            return Fraction(d)
        k += cp
        if k * M > max_rounds:
            raise NoPeriod("coalesced synchronisation did not settle")


def two_bw_lambda(prof, st, part: Partition, M: int, sync: int, max_rounds: int = MAX_ROUNDS) -> Fraction:
    """Exact steady-state time per iteration (M micro-batches) of the 2BW pipeline."""
    ing = model_ingredients(prof, st, part, sync)
    sched = Schedule(ing)
    j0, c, D = steady_state(sched, max_rounds)
    lam = Fraction(M * D, c)
    for s in range(part.S):
        if len(part.W[s]) >= 2:
            lam = max(lam, _coalesced_chain_slope(sched, s, M, ing.ar[s], j0, c, D, max_rounds))
    return lam


def two_bw_time_ns_cycles(prof, st, part: Partition, M: int, sync: int) -> int:
    """ceil of the 2BW time per iteration without waiting for the periodic regime (R-2):
    ceil(M * lambda_compute) from the max cycle ratio of the 1F1B event graph with the per-mini-batch
    synchronisation removed (durations scaled by M), and the coalesced chain's own rate d (nothing
    waits for it, so its slope is max(M lambda_compute, d) by the backlog argument above)."""
    from .cycle_ratio import ceil_max_cycle_ratio
    ing = model_ingredients(prof, st, part, sync)
    sync_d = [ing.ar[s] for s in range(part.S) if len(part.W[s]) >= 2]
    ing.ar = [0] * part.S
    return max([ceil_max_cycle_ratio(prof, st, part, ing, scale=M)] + sync_d)


# --- GPIPE / DAPPLE: one flushed iteration -------------------------------------------------------
def op_list(schedule: int, S: int, s: int, M: int) -> List[Tuple[str, int]]:
    """The operation list of a worker of stage s (reading F-3)."""
    if schedule == GPIPE:
        return [("F", k) for k in range(M)] + [("B", k) for k in range(M)]
    n = min(S - s, M)
    ops = [("F", k) for k in range(n)]
    for j in range(M):
        ops.append(("B", j))
        if j + n < M:
            ops.append(("F", j + n))
    return ops


def _op_duration(ing: Ingredients, s: int, w: int, kind: str, recompute: bool) -> int:
    if kind == "F":
        return ing.Fd[s][w]
    return ing.Bd[s][w] + (ing.Fd[s][w] if recompute else 0)


def flush_events(prof, st, part: Partition, schedule: int, M: int, recompute: bool, sync: int):
    """Ready-driven execution of one flushed iteration. Returns (end of every op, the makespan)."""
    ing = model_ingredients(prof, st, part, sync)
    S = part.S
    lists = {(s, w): op_list(schedule, S, s, M) for s in range(S) for w in part.W[s]}
    pos = {k: 0 for k in lists}
    wfree = {w: 0 for s in range(S) for w in part.W[s]}
    end: Dict[Tuple[str, int, int, int], int] = {}          # (kind, s, w, k) -> finish
    fdone: Dict[Tuple[int, int], int] = {}                   # forward boundary s of micro-batch k
    bdone: Dict[Tuple[int, int], int] = {}                   # backward boundary s of micro-batch k
    next_f, next_b = [0] * max(S - 1, 0), [0] * max(S - 1, 0)
    link_free: Dict[Tuple[int, int], int] = {}

    def ready(s: int, kind: str, k: int) -> Optional[int]:
        if kind == "F":
            return 0 if s == 0 else fdone.get((s - 1, k))
        return 0 if s == S - 1 else bdone.get((s, k))

    def boundary(bar: int, transfers) -> int:
        done = bar
        for (u, v, d) in transfers:
            start = max(bar, link_free.get((u, v), 0))
            link_free[(u, v)] = start + d
            done = max(done, start + d)
        return done

    while True:
        progress = False
        for (s, w), ops in lists.items():
            while pos[(s, w)] < len(ops):
                kind, k = ops[pos[(s, w)]]
                t = ready(s, kind, k)
                if t is None:
                    break
                start = max(wfree[w], t)
                wfree[w] = start + _op_duration(ing, s, w, kind, recompute)
                end[(kind, s, w, k)] = wfree[w]
                pos[(s, w)] += 1
                progress = True
        for s in range(S - 1):
            while next_f[s] < M and all(("F", s, w, next_f[s]) in end for w in part.W[s]):
                k = next_f[s]
                fdone[(s, k)] = boundary(max(end[("F", s, w, k)] for w in part.W[s]), ing.fwd[s])
                next_f[s] += 1
                progress = True
            while next_b[s] < M and all(("B", s + 1, w, next_b[s]) in end for w in part.W[s + 1]):
                k = next_b[s]
                bdone[(s, k)] = boundary(max(end[("B", s + 1, w, k)] for w in part.W[s + 1]), ing.bwd[s])
                next_b[s] += 1
                progress = True
        if not progress:
            break
    if any(pos[k] < len(ops) for k, ops in lists.items()):
        raise RuntimeError("flushed schedule deadlocked")
    T = 0
    for s in range(S):
        last = max(end[("B", s, w, M - 1)] for w in part.W[s])
        T = max(T, last + (ing.ar[s] if len(part.W[s]) >= 2 else 0))
    return end, T


def flush_makespan(prof, st, part: Partition, schedule: int, M: int, recompute: bool = False,
                   sync: int = RING) -> int:
    return flush_events(prof, st, part, schedule, M, recompute, sync)[1]


def flush_makespan_dag(prof, st, part: Partition, schedule: int, M: int, recompute: bool = False,
                       sync: int = RING) -> int:
    """The same makespan as the longest path of the explicit event DAG of the iteration (node weight =
    duration): worker-order edges, data edges through boundary barriers, FIFO edges on each link.
    Independent of ``flush_events`` (no ready-driven execution); for tiny instances."""
    import networkx as nx
    ing = model_ingredients(prof, st, part, sync)
    S = part.S
    g = nx.DiGraph()
    g.add_node("src", dur=0)
    g.add_node("end", dur=0)
    for s in range(S):
        for w in part.W[s]:
            ops = op_list(schedule, S, s, M)
            prev = "src"
            for (kind, k) in ops:
                n = ("op", kind, s, w, k)
                g.add_node(n, dur=_op_duration(ing, s, w, kind, recompute))
                g.add_edge(prev, n)
                prev = n
    for s in range(S - 1):
        for direction, trans, senders, receivers, kind in (
                ("f", ing.fwd[s], (s, part.W[s]), (s + 1, part.W[s + 1]), "F"),
                ("b", ing.bwd[s], (s + 1, part.W[s + 1]), (s, part.W[s]), "B")):
            for k in range(M):
                bar = ("bar", direction, s, k)
                done = ("done", direction, s, k)
                g.add_node(bar, dur=0)
                g.add_node(done, dur=0)
                for w in senders[1]:
                    g.add_edge(("op", kind, senders[0], w, k), bar)
                g.add_edge(bar, done)
                for (u, v, d) in trans:
                    x = ("x", direction, s, u, v, k)
                    g.add_node(x, dur=d)
                    g.add_edge(bar, x)
                    g.add_edge(x, done)
                    if k > 0:
                        g.add_edge(("x", direction, s, u, v, k - 1), x)   # FIFO on the link
                for w in receivers[1]:
                    g.add_edge(done, ("op", kind, receivers[0], w, k))
    for s in range(S):
        sy = ("sync", s)
        g.add_node(sy, dur=ing.ar[s] if len(part.W[s]) >= 2 else 0)
        for w in part.W[s]:
            g.add_edge(("op", "B", s, w, M - 1), sy)
        g.add_edge(sy, "end")
    if not nx.is_directed_acyclic_graph(g):
        raise RuntimeError("event graph has a cycle: the schedule would deadlock")
    best: Dict = {}
    for n in nx.topological_sort(g):
        preds = [best[p] for p in g.predecessors(n)]
        best[n] = (max(preds) if preds else 0) + g.nodes[n]["dur"]
    return best["end"]


# --- the model as a whole ----------------------------------------------------------------------
def model_time_ns(prof, st, part: Optional[Partition], schedule: int = PIPEDREAM, sync: int = RING,
                  M: int = 1, recompute: bool = False) -> int:
    """T_ns of one partition under a schedule variant (reading F-3); UINT64_MAX if invalid."""
    if part is None:
        return U64_MAX
    if schedule == PIPEDREAM:
        return time_ns(prof, st, part, model_ingredients(prof, st, part, sync))
    if schedule == TWO_BW:
        try:
            lam = two_bw_lambda(prof, st, part, M, sync, TIME_NS_ROUNDS)
        except NoPeriod:
            return two_bw_time_ns_cycles(prof, st, part, M, sync)
        return ceil_div(lam.numerator, lam.denominator)
    if schedule in (GPIPE, DAPPLE):
        return flush_makespan(prof, st, part, schedule, M, recompute and schedule == GPIPE, sync)
    raise ValueError("unknown schedule %r" % schedule)


def score_record(prof, st, rec: bytes, schedule: int = PIPEDREAM, sync: int = RING, M: int = 1,
                 recompute: bool = False) -> int:
    return model_time_ns(prof, st, parse_record(rec, len(prof.O), len(st.f)), schedule, sync, M, recompute)
