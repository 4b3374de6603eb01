"""Oracle: Chimera's bidirectional pipelines (NEXT row f3, reading F-6). Test infrastructure only.

"Chimera effectively maps stages of the model in linear and opposite orders across two pipelines,
optimizing the execution of micro-batches. This unique configuration significantly reduces idle times
(bubbles)"; AutoPipe is applied to Chimera in Fig. 13. The
paper gives no timing model; reading F-6 makes one exact, in the frame of reading F-3
(the profile describes one micro-batch, an iteration is M micro-batches and one weight update, every
result is the time of one flushed iteration in ns):

* a Chimera partition is a partition with one worker per stage (stage s on worker w_s; idle workers
  allowed). The "down" pipeline runs stage s on w_s; the "up" pipeline runs the same stages in the
  opposite order: its stage u (the same layers as stage u) on w_{S-1-u}. Every worker holds two
  stages. A record with a replicated stage is not a Chimera partition: UINT64_MAX;
* the iteration's M micro-batches split ceil(M/2) down and floor(M/2) up; each pipeline keeps
  DAPPLE's per-stage order (1F1B with flush: min(S - s, M_p) warm-up forwards, then B(j), F(j + n)
  while j + n < M_p, then the remaining backwards; reading F-3);
* a worker interleaves its two lists by readiness: repeatedly, among the ops at the heads of every
  worker's two lists whose input has been computed, the one with the earliest start max(worker free,
  input ready) runs next; ties go to the worker of the lower down stage, then to the down pipeline
  (Chimera fills one pipeline's bubbles with the other's work);
* a boundary transfer (activation O[e_s] forward, gradient G[e_s + 1] backward, reading C-6) starts
  when its producing op has finished and its directed link is free, FIFO per directed link in the
  order the transfers are issued (the two pipelines share the links between the same workers);
* stage s's two copies (on w_s and w_{S-1-s}) synchronise their gradients after the iteration's last
  backward of both (ring all-reduce over the two workers, or the sharded parameter server; nothing to
  exchange when the two copies share a worker, the middle stage of an odd S);
* T = max over stages of (the later last backward of its two copies + its sync).
With M = 1 (no up micro-batch) and weightless layers this is DAPPLE with M = 1.
"""
from __future__ import annotations

from typing import Dict, List, Optional, Tuple

from .model import U64_MAX, Partition, allreduce_duration, parse_record, xfer

RING, PS = 0, 1
DOWN, UP = 0, 1


def dapple_list(S: int, s: int, M: int) -> List[Tuple[str, int]]:
    """DAPPLE's op order for stage s of an S-stage pipeline with M micro-batches (reading F-3)."""
    n = min(S - s, M)
    ops = [("F", k) for k in range(n)]
    for j in range(M):
        ops.append(("B", j))
        if j + n < M:
            ops.append(("F", j + n))
    return ops


def chimera_events(prof, st, part: Partition, M: int, sync: int = RING):
    """Run one iteration; returns (the executed ops in order as (worker, pipe, kind, stage, k, start,
    end), T), or (None, U64_MAX) for a record that is not a Chimera partition."""
    from .schedules import ps_duration
    S = part.S
    if any(len(ws) != 1 for ws in part.W):
        return None, U64_MAX
    L = len(prof.O)
    stages = part.stage_layers(L)
    wk = [ws[0] for ws in part.W]                       # w_s: the worker of down stage s
    Md, Mu = (M + 1) // 2, M // 2
    Mp = (Md, Mu)

    def worker(pipe: int, s: int) -> int:               # the worker of stage s of a pipeline
        return wk[s] if pipe == DOWN else wk[S - 1 - s]

    def F(w: int, s: int) -> int:
        a, e = stages[s]
        return sum(st.f[w][a:e + 1])

    def B(w: int, s: int) -> int:
        a, e = stages[s]
        return sum(st.b[w][a:e + 1])

    # per worker: its two lists (the stage it holds in each pipeline)
    lists: Dict[Tuple[int, int], List[Tuple[str, int]]] = {}
    stage_of: Dict[Tuple[int, int], int] = {}
    for g in range(S):
        w = wk[g]
        for pipe, s in ((DOWN, g), (UP, S - 1 - g)):
            lists[(w, pipe)] = dapple_list(S, s, Mp[pipe])
            stage_of[(w, pipe)] = s
    pos = {key: 0 for key in lists}
    free = {w: 0 for w in wk}
    fdone: Dict[Tuple[int, int, int], int] = {}   # (pipe, boundary s, k) -> forward transfer ends
    bdone: Dict[Tuple[int, int, int], int] = {}
    link: Dict[Tuple[int, int], int] = {}
    last_b: Dict[Tuple[int, int], int] = {}      # (pipe, stage) -> end of its last backward
    done_ops = []

    def ready(pipe: int, s: int, kind: str, k: int) -> Optional[int]:
        if kind == "F":
            return 0 if s == 0 else fdone.get((pipe, s - 1, k))
        return 0 if s == S - 1 else bdone.get((pipe, s, k))

    def send(u: int, v: int, t: int, d: int) -> int:
        start = max(t, link.get((u, v), 0))
        link[(u, v)] = start + d
        return start + d

    total = sum(len(x) for x in lists.values())
    for _ in range(total):
        best = None
        for w in wk:                                   # workers in down-stage order
            for pipe in (DOWN, UP):
                ops = lists[(w, pipe)]
                if pos[(w, pipe)] >= len(ops):
                    continue
                kind, k = ops[pos[(w, pipe)]]
                s = stage_of[(w, pipe)]
                t = ready(pipe, s, kind, k)
                if t is None:
                    continue
                start = max(free[w], t)
                if best is None or start < best[0]:
                    best = (start, w, pipe, kind, s, k)
        if best is None:
            raise RuntimeError("Chimera schedule deadlocked")
        start, w, pipe, kind, s, k = best
        end = start + (F(w, s) if kind == "F" else B(w, s))
        free[w] = end
        pos[(w, pipe)] += 1
        done_ops.append((w, pipe, kind, s, k, start, end))
        if kind == "F" and s < S - 1:
            e = stages[s][1]
            u, v = worker(pipe, s), worker(pipe, s + 1)
            fdone[(pipe, s, k)] = send(u, v, end, xfer(prof.O[e], st.tau[u][v]))
        if kind == "B":
            last_b[(pipe, s)] = end
            if s > 0:
                e = stages[s - 1][1]
                u, v = worker(pipe, s), worker(pipe, s - 1)
                bdone[(pipe, s - 1, k)] = send(u, v, end, xfer(prof.G[e + 1], st.tau[u][v]))
    T = 0
    for s in range(S):
        a, e = stages[s]
        fin = max(last_b.get((DOWN, s), 0), last_b.get((UP, s), 0))
        pair = sorted({wk[s], wk[S - 1 - s]})
        if len(pair) == 2:
            fin += ps_duration(prof.P, a, e, pair, st.tau) if sync == PS else allreduce_duration(prof.P, a, e, pair, st.tau)
        T = max(T, fin)
    return done_ops, T


def time_ns(prof, st, part: Optional[Partition], M: int, sync: int = RING) -> int:
    if part is None:
        return U64_MAX
    return chimera_events(prof, st, part, M, sync)[1]


def score_record(prof, st, rec: bytes, M: int, sync: int = RING) -> int:
    return time_ns(prof, st, parse_record(rec, len(prof.O), len(st.f)), M, sync)
