"""Oracle cross-check: max cycle ratio of the explicit timed event graph (SPEC.md §3-4).
Test infrastructure only; used on tiny instances to pin ``sim.simulate``.

The schedule of SPEC §3 is a timed event graph: node v(j) finishes at max over its predecessors
u(j - tokens(u,v)) plus its own duration. For such a graph the asymptotic time per round of every
node is the largest (sum of node durations) / (sum of edge tokens) over the elementary cycles that
reach it (max-plus spectral theory), so lambda = the maximum cycle ratio over all elementary cycles.
Cycles are enumerated with networkx.simple_cycles (Johnson's algorithm).

Nodes (per round j, as in sim.Schedule): F[s,w] = F_{s,w}(j+n_s), B[s,w] = B_{s,w}(j), the barrier
and completion of each boundary, one node per transfer, one all-reduce node per replicated stage.
"""
from __future__ import annotations

from fractions import Fraction

import networkx as nx

from typing import Optional

from .model import Ingredients, Partition, ingredients


def event_graph(prof, st, part: Partition, ing: Optional[Ingredients] = None) -> nx.DiGraph:
    ing = ing if ing is not None else ingredients(prof, st, part)
    S = part.S
    g = nx.DiGraph()

    def node(name, dur):
        g.add_node(name, dur=dur)

    def edge(u, v, tokens):
        g.add_edge(u, v, tokens=tokens)

    for s in range(S):
        for w in part.W[s]:
            node(("F", s, w), ing.Fd[s][w])
            node(("B", s, w), ing.Bd[s][w])
            # worker order: ... F(j-1+n) -> B(j) -> F(j+n) -> B(j+1) ...
            edge(("F", s, w), ("B", s, w), 1)
            edge(("B", s, w), ("F", s, w), 0)
        if len(part.W[s]) >= 2:
            node(("AR", s), ing.ar[s])
            edge(("AR", s), ("AR", s), 1)
            for w in part.W[s]:
                edge(("B", s, w), ("AR", s), 0)
    for s in range(S - 1):
        # forward boundary s, mini-batch j + n_s (round j)
        node(("Xf", s), 0)
        node(("Df", s), 0)
        for w in part.W[s]:
            edge(("F", s, w), ("Xf", s), 0)
        if not ing.fwd[s]:
            edge(("Xf", s), ("Df", s), 0)
        for (u, v, d) in ing.fwd[s]:
            t = ("Tf", s, u, v)
            node(t, d)
            edge(("Xf", s), t, 0)
            edge(t, t, 1)                      # FIFO link: one transfer per round
            edge(t, ("Df", s), 0)
        # F_{s+1}(j + n_{s+1}) needs boundary s of mini-batch j + n_{s+1} = (j-1) + n_s: 1 token
        for w in part.W[s + 1]:
            edge(("Df", s), ("F", s + 1, w), 1)
        # backward boundary s, mini-batch j (round j)
        node(("Xb", s), 0)
        node(("Db", s), 0)
        for w in part.W[s + 1]:
            edge(("B", s + 1, w), ("Xb", s), 0)
        if not ing.bwd[s]:
            edge(("Xb", s), ("Db", s), 0)
        for (u, v, d) in ing.bwd[s]:
            t = ("Tb", s, u, v)
            node(t, d)
            edge(("Xb", s), t, 0)
            edge(t, t, 1)
            edge(t, ("Db", s), 0)
        for w in part.W[s]:
            edge(("Db", s), ("B", s, w), 0)
    return g


def ceil_max_cycle_ratio(prof, st, part: Partition, ing: Optional[Ingredients] = None, scale: int = 1) -> int:
    """ceil(lambda) without enumerating cycles: the smallest integer theta such that no cycle has
    sum(durations) - theta * sum(tokens) > 0, found by binary search on theta with a Bellman-Ford
    positive-cycle test (longest paths from a virtual source). Used by ``sim.time_ns`` when the
    simulation's transient is too long to wait for (two near-equal cycle ratios). ``scale`` = k
    returns ceil(k * lambda) instead (durations scaled by k; 2BW's iteration of k micro-batches)."""
    g = event_graph(prof, st, part, ing)
    nodes = list(g.nodes)
    pos = {v: i for i, v in enumerate(nodes)}
    dur = [g.nodes[v]["dur"] * scale for v in nodes]
    edges = [(pos[u], pos[v], g.edges[u, v]["tokens"]) for u, v in g.edges]

    def positive_cycle(theta: int) -> bool:
        d = [0] * len(nodes)
        for _ in range(len(nodes)):
            changed = False
            for (u, v, tok) in edges:
                nd = d[u] + dur[v] - theta * tok
                if nd > d[v]:
                    d[v] = nd
                    changed = True
            if not changed:
                return False
        return True

    lo, hi = -1, max(1, sum(dur))        # lambda <= sum of all durations (every cycle has >= 1 token)
    while hi - lo > 1:
        mid = (lo + hi) // 2
        if positive_cycle(mid):
            lo = mid
        else:
            hi = mid
    return hi


def max_cycle_ratio(prof, st, part: Partition) -> Fraction:
    g = event_graph(prof, st, part)
    best = None
    for cyc in nx.simple_cycles(g):
        dur = sum(g.nodes[v]["dur"] for v in cyc)
        tok = sum(g.edges[cyc[i], cyc[(i + 1) % len(cyc)]]["tokens"] for i in range(len(cyc)))
        if tok == 0:
            raise ValueError("zero-token cycle: the schedule would deadlock")
        r = Fraction(dur, tok)
        if best is None or r > best:
            best = r
    return best
