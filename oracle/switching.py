"""Oracle: the switching cost of a new partition as time. Test infrastructure only.

The paper names two costs of switching the work partition: "we need to pause the
training. Meanwhile, the flow line requires a restart phase, i.e., startup starts in Figure 2,
which brings bubbles", and the switch moves layer weights between workers. Its
arbiter's reward is "the training speed of one iteration" with "the normalized switching cost"
(PAPER.md:924-927), which it learns with a network; this module defines the analytic replacement
(reading F-2):

* refill_ns(p)   = max(0, C_{S-1} - S * T_ns(p)), where C_k is the time mini-batch k's backward pass
                   leaves stage 0 (every replica done) in the static 1F1B schedule of p started
                   empty at time 0 — the startup state of Fig. 2, measured over the first S
                   mini-batches (the n_0 = S admitted before stage 0's first backward), in excess
                   of S steady-state periods;
* migrate_ns(p|c)= max over workers w of the sum of the messages w receives: for every stage s' of
                   the current partition c that covers some of w's new layers and does not hold w,
                   one message of the weight bytes of those layers from the cheapest holder
                   (xfer(bytes, min over u in W_c[s'] of tau[u][w])); a worker receives its
                   messages one after another, different workers in parallel;
* both are 0 when p gives every worker the same layer set as c (nothing switches);
* reward_ns      = T_ns(p) + ceil((refill_ns + migrate_ns) / H), H >= 1 the number of iterations
                   the switch is amortised over.

Everything is computed by the definitions: C_k is read off the event-by-event simulation of
``sim.Schedule`` (the same schedule that defines T_ns), the messages by walking layers one by one.
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

from .model import U64_MAX, Partition, ceil_div, ingredients, parse_record, xfer
from .neighbourhood import layer_sets
from .sim import Schedule, time_ns


def startup_completions(prof, st, p: Partition, K: int) -> List[int]:
    """C_0 .. C_{K-1}: when the backward pass of mini-batch k completes on every replica of stage 0,
    in the 1F1B schedule of p started from an empty pipeline at time 0 (Fig. 2)."""
    sched = Schedule(ingredients(prof, st, p))
    sched.run_to(K - 1)  # round k holds B(k) of every stage
    return [max(sched.B[(0, w, k)] for w in p.W[0]) for k in range(K)]


def refill_ns(prof, st, p: Partition, T: int) -> int:
    """Startup bubbles of p: the first S mini-batches' completion time in excess
    of S steady-state periods T, never negative."""
    C = startup_completions(prof, st, p, p.S)
    return max(0, C[-1] - p.S * T)


def gained_messages(prof, st, new: Partition, old: Partition) -> List[List[Tuple[int, int]]]:
    """Per worker w, its weight messages (bytes, duration) under new vs old:
    the layers of w's new stage are grouped by the old stage that holds them; a group held by a stage
    w belonged to needs nothing, any other group is one message from its cheapest holder."""
    L, N = len(prof.O), len(st.f)
    old_stage_of_layer = [None] * L
    for s, (a, e) in enumerate(old.stage_layers(L)):
        for l in range(a, e + 1):
            old_stage_of_layer[l] = s
    out: List[List[Tuple[int, int]]] = [[] for _ in range(N)]
    for s, (a, e) in enumerate(new.stage_layers(L)):
        for w in new.W[s]:
            groups = {}
            for l in range(a, e + 1):  # layer by layer
                so = old_stage_of_layer[l]
                if w in old.W[so]:
                    continue
                groups[so] = groups.get(so, 0) + prof.P[l]
            for so in sorted(groups):
                tau = min(st.tau[u][w] for u in old.W[so])
                out[w].append((groups[so], xfer(groups[so], tau)))
    return out


def migrate_ns(prof, st, new: Partition, old: Partition) -> int:
    msgs = gained_messages(prof, st, new, old)
    return max([sum(d for _, d in m) for m in msgs] + [0])


def switch_reward(prof, st, rec: bytes, current: Partition, horizon: int) -> Tuple[int, int, int, int]:
    """(T_ns, refill_ns, migrate_ns, reward_ns) of one proposal; all UINT64_MAX if it is invalid."""
    L, N = len(prof.O), len(st.f)
    p = parse_record(rec, L, N)
    if p is None:
        return (U64_MAX,) * 4
    T = time_ns(prof, st, p)
    if layer_sets(p, L, N) == layer_sets(current, L, N):
        return T, 0, 0, T
    R = refill_ns(prof, st, p, T)
    M = migrate_ns(prof, st, p, current)
    return T, R, M, T + ceil_div(R + M, horizon)


def switch_rewards(prof, st, records: Sequence[bytes], current: bytes, horizon: int
                   ) -> List[Tuple[int, int, int, int]]:
    L, N = len(prof.O), len(st.f)
    cur: Optional[Partition] = parse_record(current, L, N)
    if cur is None:
        raise ValueError("invalid current partition")  # the C-ABI returns AUTOPIPE_E_INVAL
    if horizon < 1:
        raise ValueError("horizon must be >= 1")
    return [switch_reward(prof, st, rec, cur, horizon) for rec in records]
