"""Oracle: event-by-event simulation of the static 1F1B schedule (SPEC.md §3). Test infrastructure only.

Follows the schedule of PipeDream-style 1F1B with weight stashing (Fig. 1c at
144-163, Fig. 2 at 463-475 with the text at 567-580; weight stashing PAPER.md:320-331, 478-483):

* every worker runs its fixed operation list F(0..n_s-1), B(0), F(n_s), B(1), ... (n_s = S - s);
* an operation starts when its worker is free and its input has arrived;
* each stage boundary is a barrier followed by FIFO transfers on directed links;
* replicated stages all-reduce their gradients every mini-batch; nothing waits for it.

The simulation is generic: it repeatedly executes whichever operation is ready; it does not use the
closed form of SPEC §4. The period is found exactly: the events are grouped into rounds
(round j = B(j) and F(j + n_s) of every worker of stage s, plus the transfers those feed); the
round-(j+1) times are a max-plus function of the round-j times, so the first time the vector of
round times repeats up to a constant shift (R(j) = R(j') + D) the schedule is periodic from j'
on and lambda = D / (j - j'). All-reduce chains feed nothing, so they may fall behind without bound;
each is checked separately (see ``_allreduce_slope``). The result is an exact Fraction.
"""
from __future__ import annotations

from fractions import Fraction
from typing import Dict, List, Optional, Tuple

from .model import U64_MAX, Ingredients, Partition, ceil_div, ingredients, parse_record

MAX_ROUNDS = 10**6
# time_ns waits this many rounds for the periodic regime before taking ceil(lambda) from the max
# cycle ratio of the same event graph instead (cycle_ratio.ceil_max_cycle_ratio; reading R-2)
TIME_NS_ROUNDS = 4000


class NoPeriod(RuntimeError):
    """The schedule did not become periodic within the allowed number of rounds."""


class Schedule:
    """The timed static 1F1B schedule of one partition, simulated lazily round by round."""

    def __init__(self, ing: Ingredients):
        self.ing = ing
        S = ing.S
        self.S = S
        self.n = [S - s for s in range(S)]
        self.workers = [(s, w) for s in range(S) for w in ing.W[s]]
        self.F: Dict[Tuple[int, int, int], int] = {}    # (s, w, k) -> finish of F_{s,w}(k)
        self.B: Dict[Tuple[int, int, int], int] = {}    # (s, w, k) -> finish of B_{s,w}(k)
        self.Fstart: Dict[Tuple[int, int, int], int] = {}
        self.Bstart: Dict[Tuple[int, int, int], int] = {}
        self.fbar: Dict[Tuple[int, int], int] = {}      # forward boundary s of k: barrier time
        self.fdone: Dict[Tuple[int, int], int] = {}     # ... completion
        self.bbar: Dict[Tuple[int, int], int] = {}
        self.bdone: Dict[Tuple[int, int], int] = {}
        self.fx: Dict[Tuple[int, int, int, int], int] = {}  # (s, u, v, k) -> end of that transfer
        self.bx: Dict[Tuple[int, int, int, int], int] = {}
        self.ar: Dict[Tuple[int, int], int] = {}        # (s, k) -> end of AR_s(k)
        self.link_free: Dict[Tuple[int, int], int] = {}
        self.wfree: Dict[int, int] = {w: 0 for _, w in self.workers}
        self.pos: Dict[Tuple[int, int], int] = {sw: 0 for sw in self.workers}  # index in op list
        self.next_f = [0] * max(S - 1, 0)
        self.next_b = [0] * max(S - 1, 0)
        self.next_ar = [0] * S
        self.rounds_done = -2

    # -- the fixed per-worker operation list (SPEC §3 "worker order") ---------------------
    def op_at(self, s: int, i: int) -> Tuple[str, int]:
        """The i-th operation of a worker of stage s: F(0..n-1), then B(j), F(j+n) for j = 0, 1, ..."""
        n = self.n[s]
        if i < n:
            return ("F", i)
        j, odd = divmod(i - n, 2)
        return ("B", j) if odd == 0 else ("F", j + n)

    def round_of(self, s: int, op: Tuple[str, int]) -> int:
        kind, k = op
        return k if kind == "B" else max(k - self.n[s], -1)

    # -- readiness ----------------------------------------------------------------------
    def ready_time(self, s: int, op: Tuple[str, int]) -> Optional[int]:
        kind, k = op
        if kind == "F":
            return 0 if s == 0 else self.fdone.get((s - 1, k))
        return 0 if s == self.S - 1 else self.bdone.get((s, k))

    def _try_boundaries(self) -> bool:
        ing, progress = self.ing, False
        for s in range(self.S - 1):
            # forward boundary s: barrier over all F_{s,.}(k), then FIFO transfers W_s -> W_{s+1}
            while True:
                k = self.next_f[s]
                ends = [self.F.get((s, w, k)) for w in ing.W[s]]
                if any(x is None for x in ends):
                    break
                bar = max(ends)
                self.fbar[(s, k)] = bar
                done = bar
                for (u, v, d) in ing.fwd[s]:
                    start = max(bar, self.link_free.get((u, v), 0))
                    self.link_free[(u, v)] = start + d
                    self.fx[(s, u, v, k)] = start + d
                    done = max(done, start + d)
                self.fdone[(s, k)] = done
                self.next_f[s] += 1
                progress = True
            # backward boundary s: barrier over all B_{s+1,.}(k), then transfers W_{s+1} -> W_s
            while True:
                k = self.next_b[s]
                ends = [self.B.get((s + 1, w, k)) for w in ing.W[s + 1]]
                if any(x is None for x in ends):
                    break
                bar = max(ends)
                self.bbar[(s, k)] = bar
                done = bar
                for (u, v, d) in ing.bwd[s]:
                    start = max(bar, self.link_free.get((u, v), 0))
                    self.link_free[(u, v)] = start + d
                    self.bx[(s, u, v, k)] = start + d
                    done = max(done, start + d)
                self.bdone[(s, k)] = done
                self.next_b[s] += 1
                progress = True
        for s in range(self.S):
            if len(ing.W[s]) < 2:
                continue
            while True:
                k = self.next_ar[s]
                ends = [self.B.get((s, w, k)) for w in ing.W[s]]
                if any(x is None for x in ends):
                    break
                prev = self.ar.get((s, k - 1), 0)
                self.ar[(s, k)] = max(max(ends), prev) + ing.ar[s]
                self.next_ar[s] += 1
                progress = True
        return progress

    def run_to(self, target: int) -> None:
        """Execute every operation of rounds <= target (and whatever boundaries they complete)."""
        if target <= self.rounds_done:
            return
        ing = self.ing
        while True:
            progress = False
            for (s, w) in self.workers:
                while True:
                    op = self.op_at(s, self.pos[(s, w)])
                    if self.round_of(s, op) > target:
                        break
                    t = self.ready_time(s, op)
                    if t is None:
                        break
                    kind, k = op
                    start = max(self.wfree[w], t)
                    if kind == "F":
                        end = start + ing.Fd[s][w]
                        self.Fstart[(s, w, k)] = start
                        self.F[(s, w, k)] = end
                    else:
                        end = start + ing.Bd[s][w]
                        self.Bstart[(s, w, k)] = start
                        self.B[(s, w, k)] = end
                    self.wfree[w] = end
                    self.pos[(s, w)] += 1
                    progress = True
            if self._try_boundaries():
                progress = True
            if not progress:
                break
        for (s, w) in self.workers:
            if self.round_of(s, self.op_at(s, self.pos[(s, w)])) <= target:
                raise RuntimeError("static 1F1B schedule deadlocked")  # impossible for S >= 1
        self.rounds_done = target

    def components(self) -> List[List[Tuple[int, int]]]:
        """Groups of workers whose events depend on each other. For S >= 2 every worker is coupled to
        every other through the stage barriers and the 1F1B order (one group). For S = 1 there is no
        boundary: each replica runs F, B, F, B, ... on its own and is its own group."""
        if self.S == 1:
            return [[sw] for sw in self.workers]
        return [list(self.workers)]

    def round_vector(self, j: int, comp: Optional[List[Tuple[int, int]]] = None) -> List[int]:
        """All event times of round j: F_{s,w}(j+n_s), B_{s,w}(j), and the boundary events they feed."""
        ing, vec = self.ing, []
        for (s, w) in (self.workers if comp is None else comp):
            vec.append(self.F[(s, w, j + self.n[s])])
            vec.append(self.B[(s, w, j)])
        for s in range(self.S - 1):
            k = j + self.n[s]
            vec.append(self.fbar[(s, k)])
            vec.append(self.fdone[(s, k)])
            vec.extend(self.fx[(s, u, v, k)] for (u, v, _) in ing.fwd[s])
            vec.append(self.bbar[(s, j)])
            vec.append(self.bdone[(s, j)])
            vec.extend(self.bx[(s, u, v, j)] for (u, v, _) in ing.bwd[s])
        return vec

    def ensure(self, j: int) -> None:
        if j > self.rounds_done:
            self.run_to(max(j, 2 * self.rounds_done + 8))


def compute_period(sched: Schedule, comp=None, max_rounds: int = MAX_ROUNDS) -> Tuple[int, int, int]:
    """First repeat of the normalised round vector: returns (j0, c, D), lambda_compute = D / c."""
    seen: Dict[tuple, Tuple[int, int]] = {}
    j = 0
    while j <= max_rounds:
        sched.ensure(j + 1)
        vec = sched.round_vector(j, comp)
        m = min(vec)
        key = tuple(x - m for x in vec)
        if key in seen:
            j0, m0 = seen[key]
            return j0, j - j0, m - m0
        seen[key] = (j, m)
        j += 1
    raise NoPeriod("no periodicity within %d rounds" % max_rounds)


def _allreduce_slope(sched: Schedule, s: int, j0: int, c: int, lam_c: Fraction,
                     max_rounds: int = MAX_ROUNDS) -> Fraction:
    """Asymptotic slope of the all-reduce chain of stage s (SPEC §3).

    AR(k) = max(Bmax(k), AR(k-1)) + d. Let o(k) = AR(k) - Bmax(k) - d >= 0 (its backlog). Once the
    compute events are periodic (from j0, period c), the map o(k) -> o(k+c) is monotone, so:
    * o(k+c) == o(k): the chain repeats with the compute pattern, slope lambda_c;
    * o > 0 over the whole period (so every step adds exactly d) and o(k+c) > o(k): the backlog
      never clears again (monotonicity), slope d.
    One of the two happens after finitely many periods (Lindley's recursion)."""
    d = sched.ing.ar[s]
    W = sched.ing.W[s]

    def o(k: int) -> int:
        return sched.ar[(s, k)] - max(sched.B[(s, w, k)] for w in W) - d

    k = j0
    while True:
        sched.ensure(k + c + 1)
        if o(k + c) == o(k):
            return lam_c
        if all(o(i) > 0 for i in range(k + 1, k + c + 1)) and o(k + c) > o(k):
            return Fraction(d)
        k += c
        if k > max_rounds:
            raise NoPeriod("all-reduce chain did not settle within %d rounds" % max_rounds)


def steady_state(sched: Schedule, max_rounds: int = MAX_ROUNDS) -> Tuple[int, int, int]:
    """(j0, c, D): the compute events of ``sched`` are periodic from round j0 with period c and shift D
    (lambda_compute = D / c), combining the independent groups of ``Schedule.components``."""
    periods = [compute_period(sched, comp, max_rounds) for comp in sched.components()]
    if len(periods) == 1:
        return periods[0]
    # S = 1 with replicas: each replica runs back to back from t = 0, so B_w(k) = (k+1) X_w exactly
    # (its round vector repeats from round 0 with period 1); the slowest replica is the max at
    # every k, hence max_w B_w(k) is periodic from 0 with period 1 and shift max_w X_w.
    assert all(j0 == 0 and c == 1 for (j0, c, _) in periods)
    return 0, 1, max(D for (_, _, D) in periods)


def simulate(prof, st, part: Partition, max_rounds: int = MAX_ROUNDS, ing: Optional[Ingredients] = None
             ) -> Fraction:
    """Exact steady-state time per mini-batch lambda (SPEC §3 'Result'), as a Fraction.
    Raises NoPeriod if the periodic regime is not reached within max_rounds rounds. ``ing`` replaces
    the ingredients of SPEC §2-3 (used by the PS synchronisation of oracle/schedules.py)."""
    sched = Schedule(ing if ing is not None else ingredients(prof, st, part))
    j0, c, D = steady_state(sched, max_rounds)
    lam = Fraction(D, c)
    for s in range(part.S):
        if len(part.W[s]) >= 2:
            lam = max(lam, _allreduce_slope(sched, s, j0, c, Fraction(D, c), max_rounds))
    return lam


def time_ns(prof, st, part: Optional[Partition], ing: Optional[Ingredients] = None) -> int:
    """T_ns = ceil(lambda) (reading C-7); UINT64_MAX for an invalid record."""
    if part is None:
        return U64_MAX
    try:
        lam = simulate(prof, st, part, TIME_NS_ROUNDS, ing)
    except NoPeriod:
        from .cycle_ratio import ceil_max_cycle_ratio
        return ceil_max_cycle_ratio(prof, st, part, ing)
    return ceil_div(lam.numerator, lam.denominator)


def score_record(prof, st, rec: bytes) -> int:
    return time_ns(prof, st, parse_record(rec, len(prof.O), len(st.f)))
