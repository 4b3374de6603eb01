"""Pins of the oracle's event simulation against what the paper and mathematics fix (CPU only).

Each test names the passage or fact it pins. A plausible mistake in the simulation (wrong in-flight
count, a dropped transfer, a transposed link, B waiting for the wrong boundary, rounding in the wrong
place) fails at least one of them.
"""
import os
from fractions import Fraction
from math import comb

import numpy as np
import pytest

import workloads as W
from oracle.model import Partition, ceil_div, parse_record, switch_bytes, xfer
from oracle.sim import Schedule, simulate, time_ns
from oracle.model import ingredients

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    out = {}
    with open(os.path.join(GOLD, name)) as fh:
        for line in fh:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(None, 1)
            out[k] = v
    return out


def uniform(L, S, f, b, c, N=None, fs=10**6):
    """L identical layers, one worker per stage, even split; every boundary transfer lasts c ns."""
    N = N or S
    # one byte per ns of transfer at tau = 1e6 fs/B
    prof = W.Profile("u", [c] * L, [c] * L, [0] * L, [f] * L, [b] * L)
    st = W.State([[f] * L for _ in range(N)], [[b] * L for _ in range(N)],
                 [[0 if u == v else fs for v in range(N)] for u in range(N)])
    m = L // S
    return prof, st, Partition(S, [m * (i + 1) - 1 for i in range(S - 1)], [[s] for s in range(S)])


# --------------------------------------------------------------------------------------------
# worked examples of the paper
# --------------------------------------------------------------------------------------------

def test_fig2_ideal_pipeline():
    """PAPER.md:463-475 + 567-580: 4 workers, F=1, B=2, no comm -> period 3, 100% utilisation,
    worker 1 runs F1 F2 F3 F4 B1 F5 B2 F6 B3 F7 B4, and the startup fills one worker per time unit."""
    g = _golden("fig2_pipedream_ideal.txt")
    S, Fu, Bu = int(g["workers"]), int(g["F"]), int(g["B"])
    prof, st, part = uniform(S, S, Fu, Bu, int(g["comm"]))
    assert simulate(prof, st, part) == int(g["steady_period"])
    sched = Schedule(ingredients(prof, st, part))
    sched.run_to(8)
    # worker-1 order: sort its recorded operations by start time
    ops = [(t, "F%d" % (k + 1)) for (s, w, k), t in sched.Fstart.items() if s == 0]
    ops += [(t, "B%d" % (k + 1)) for (s, w, k), t in sched.Bstart.items() if s == 0]
    order = [name for _, name in sorted(ops)][:11]
    assert order == g["worker1_order"].split()
    # startup state: F of mini-batch 1 reaches worker s+1 at time s (one unit per worker)
    for s in range(S):
        assert sched.Fstart[(s, s, 0)] == s * Fu
    # steady state: every worker busy F+B per period = 100% utilisation
    util = Fraction(Fu + Bu, simulate(prof, st, part))
    assert util == int(g["utilisation"])


def test_fig1c_two_workers():
    """two workers, two layers, F = B -> one mini-batch per F + B."""
    g = _golden("fig1c_two_workers.txt")
    prof, st, part = uniform(2, 2, int(g["F"]), int(g["B"]), int(g["comm"]))
    assert simulate(prof, st, part) == int(g["steady_period"])


@pytest.mark.parametrize("row", [l.split() for l in open(os.path.join(GOLD, "uniform_closed_form.txt"))
                                 if l.strip() and not l.startswith("#")])
def test_uniform_closed_form(row):
    """lambda = max(m(f+b), (L(f+b)+2(S-1)c)/S, c) for uniform layers (Observation 3)."""
    L, S, f, b, c = map(int, row[:5])
    expect = Fraction(row[5])
    m = L // S
    assert expect == max(Fraction(m * (f + b)), Fraction(L * (f + b) + 2 * (S - 1) * c, S), Fraction(c))
    assert simulate(*uniform(L, S, f, b, c)) == expect


def test_two_stage_comm_example():
    """2 stages, F = B = cf = cb = 1: the segment cycle F0 -> cf -> F1 -> B1 -> cb -> B0 carries 2
    mini-batches, so lambda = (1+1+1+1+1+1)/2 = 3."""
    assert simulate(*uniform(2, 2, 1, 1, 1)) == 3


# --------------------------------------------------------------------------------------------
# special cases that reduce to something textbook
# --------------------------------------------------------------------------------------------

def test_single_stage_is_serial_time():
    """S = 1, r = 1: no pipeline, one worker runs F and B of every layer back to back."""
    rng = np.random.default_rng(3)
    for _ in range(20):
        L = int(rng.integers(1, 12))
        prof = W.random_profile(L, rng)
        st = W.random_state_small(prof, 3, rng)
        w = int(rng.integers(0, 3))
        part = Partition(1, [], [[w]])
        assert simulate(prof, st, part) == sum(st.f[w]) + sum(st.b[w])


def test_data_parallel_allreduce():
    """S = 1, r = 2 (pure data parallelism, Fig. 1a): each replica takes half of every mini-batch,
    the ring all-reduce moves 2(r-1) chunks of ceil(P/2) bytes:
    lambda = max(ceil(F/2) + ceil(B/2), 2 * ceil(ceil(P/2) * tau / 1e6))."""
    for F, B, P, tau in [(7, 9, 1001, 10**6), (100, 200, 10, 10**6), (5, 5, 999, 3 * 10**6),
                         (1, 1, 0, 10**6), (10, 11, 10**9, 800_000)]:
        prof = W.Profile("dp", [0], [0], [P], [F], [B])
        st = W.State([[F], [F]], [[B], [B]], [[0, tau], [tau, 0]])
        expect = max(ceil_div(F, 2) + ceil_div(B, 2), 2 * ceil_div(ceil_div(P, 2) * tau, 10**6))
        assert simulate(prof, st, Partition(1, [], [[0, 1]])) == expect


def test_data_parallel_slowest_replica():
    """S = 1, r = 3 on heterogeneous workers: the slowest replica sets the pace."""
    prof = W.Profile("dp", [0, 0], [0, 0], [0, 0], [3, 4], [5, 6])
    st = W.State([[3, 4], [6, 8], [1, 1]], [[5, 6], [10, 12], [1, 1]], [[0] * 3] * 3)
    # worker 1: ceil(14/3) + ceil(22/3) = 5 + 8
    assert simulate(prof, st, Partition(1, [], [[0, 1, 2]])) == 13


def _minmax_partition(cost, S):
    """Textbook linear partition (min over contiguous S-splits of the max part sum), by DP."""
    L = len(cost)
    pre = [0]
    for c in cost:
        pre.append(pre[-1] + c)
    INF = float("inf")
    best = [[INF] * (L + 1) for _ in range(S + 1)]
    best[0][0] = 0
    for s in range(1, S + 1):
        for e in range(1, L + 1):
            for a in range(s - 1, e):
                best[s][e] = min(best[s][e], max(best[s - 1][a], pre[e] - pre[a]))
    return best[S][L]


def test_zero_comm_is_min_max_partition():
    """No communication, identical workers, one per stage, F = B/2 (Observation 3's ideal case,
    PAPER.md:567-580): the pipeline fills and the period is the bottleneck stage, so the best S-stage
    partition is the textbook min-max contiguous partition (PipeDream's zero-comm case)."""
    from oracle.search import brute_force
    rng = np.random.default_rng(5)
    for _ in range(8):
        L = int(rng.integers(2, 8))
        S = int(rng.integers(1, min(4, L) + 1))
        f = [int(x) for x in rng.integers(1, 50, size=L)]
        prof = W.Profile("z", [0] * L, [0] * L, [0] * L, f, [2 * x for x in f])
        st = W.State([f] * S, [[2 * x for x in f]] * S, [[0] * S for _ in range(S)])
        # with S workers and sum r <= S, restricting to exactly S one-worker stages:
        T, _, part, _ = brute_force(prof, st, S, S, flags=1)
        cost = [3 * x for x in f]
        if S == 1 or all(len(w) == 1 for w in part.W):
            assert T == _minmax_partition(cost, S)


def test_replicated_boundary_shards():
    """Stage 0 split over 2 replicas -> stage 1 on one worker, A = O[e] = 10 bytes: sender 0 holds
    [0,5), sender 1 holds [5,10); both go to the receiver in parallel on links 0->2 and 1->2
    (5 ns each at 1e6 fs/B). Backward G[1] = 9 bytes from worker 2 to shards [0,4), [4,9):
    4 ns to worker 0 and 5 ns to worker 1. Link 1->2 is made 3x slower: 15 ns.
    X0 = ceil(8/2) + ceil(8/2) = 8; X1 = 6; cf = 15; cb = 5;
    lambda = max(8, 6, 15, 5, ceil((8 + 6 + 15 + 5) / 2) = 17) = 17."""
    prof = W.Profile("sh", [10, 0], [0, 9], [0, 0], [8, 2], [8, 4])
    f = [[8, 2]] * 3
    b = [[8, 4]] * 3
    tau = [[0, 10**6, 10**6], [10**6, 0, 3 * 10**6], [10**6, 10**6, 0]]
    st = W.State([list(r) for r in f], [list(r) for r in b], tau)
    part = Partition(2, [0], [[0, 1], [2]])
    ing = ingredients(prof, st, part)
    assert sorted(ing.fwd[0]) == [(0, 2, 5), (1, 2, 15)]
    assert sorted(ing.bwd[0]) == [(2, 0, 4), (2, 1, 5)]
    assert simulate(prof, st, part) == 17


def test_rounding_is_per_op_and_final():
    """Reading C-7: ceil(sum/r) per replica op, ceil(bytes*tau/1e6) per transfer, ceil(lambda) once."""
    assert xfer(3, 333_334) == 2            # 1.000002 -> 2
    assert xfer(3, 333_333) == 1            # 0.999999 -> 1
    prof, st, part = uniform(3, 2, 1, 1, 0)  # stages of 1 and 2 layers: lambda = max(2, 4, 6/2)
    assert simulate(prof, st, part) == 4
    prof, st, part = uniform(8, 4, 3, 6, 5)
    assert simulate(prof, st, part) == Fraction(51, 2) and time_ns(prof, st, part) == 26


# --------------------------------------------------------------------------------------------
# invariants
# --------------------------------------------------------------------------------------------

def _terms_bounds(prof, st, part):
    ing = ingredients(prof, st, part)
    singles = [ing.Fd[s][w] + ing.Bd[s][w] for s in range(part.S) for w in part.W[s]]
    singles += ing.ar + [d for tr in ing.fwd + ing.bwd for (_, _, d) in tr]
    upper = (sum(max(ing.Fd[s].values()) + max(ing.Bd[s].values()) for s in range(part.S))
             + sum(d for tr in ing.fwd + ing.bwd for (_, _, d) in tr) + sum(ing.ar))
    return max(singles), upper


def test_invariants_random():
    """lambda >= every single term (worker F+B, each transfer, each all-reduce);
    lambda <= total compute + total comm + total all-reduce (one mini-batch alone through the pipe)."""
    rng = np.random.default_rng(11)
    for it in range(60):
        L = int(rng.integers(1, 9))
        N = int(rng.integers(1, 7))
        prof = W.random_profile(L, rng)
        st = W.random_state_small(prof, N, rng)
        for r in W.sample_records(L, N, 5, it):
            p = parse_record(bytes(r), L, N)
            if p is None:
                continue
            lam = simulate(prof, st, p)
            lo, hi = _terms_bounds(prof, st, p)
            assert lo <= lam <= hi


def _bump(obj, attr, idx, delta):
    import copy
    o = copy.deepcopy(obj)
    ref = getattr(o, attr)
    if isinstance(idx, tuple):
        ref[idx[0]][idx[1]] += delta
    else:
        ref[idx] += delta
    return o


def test_monotone():
    """More compute, more bytes, or less bandwidth (tau up) never lowers lambda."""
    rng = np.random.default_rng(12)
    for it in range(40):
        L = int(rng.integers(2, 7))
        N = int(rng.integers(2, 6))
        prof = W.random_profile(L, rng)
        st = W.random_state_small(prof, N, rng)
        recs = [bytes(r) for r in W.sample_records(L, N, 3, 100 + it)]
        for rec in recs:
            p = parse_record(rec, L, N)
            base = simulate(prof, st, p)
            l = int(rng.integers(0, L))
            w = int(rng.integers(0, N))
            u, v = [int(x) for x in rng.choice(N, 2, replace=False)]
            d = int(rng.integers(1, 500))
            assert simulate(prof, _bump(st, "f", (w, l), d), p) >= base
            assert simulate(prof, _bump(st, "b", (w, l), d), p) >= base
            assert simulate(prof, _bump(st, "tau", (u, v), 1000 * d), p) >= base
            assert simulate(_bump(prof, "O", l, 1000 * d), st, p) >= base
            assert simulate(_bump(prof, "G", l, 1000 * d), st, p) >= base
            assert simulate(_bump(prof, "P", l, 1000 * d), st, p) >= base


def test_allreduce_backlog_dominates():
    """A replicated stage whose all-reduce is slower than the pipeline period: the all-reduce chain
    falls behind forever and sets the rate (weight stashing lets compute run ahead, C-4)."""
    prof = W.Profile("ar", [0, 0], [0, 0], [10**6, 10**6], [1, 1], [1, 1])
    st = W.State([[1, 1]] * 3, [[1, 1]] * 3, [[0, 10**6, 10**6], [10**6, 0, 10**6], [10**6, 10**6, 0]])
    # stage 1 on workers {1,2}: AR = 2*ceil(ceil(1e6/2)*1e6/1e6) = 1e6; compute period is tiny
    assert simulate(prof, st, Partition(2, [0], [[0], [1, 2]])) == 10**6


# --------------------------------------------------------------------------------------------
# record validity (SPEC §2) and switch bytes (SPEC §6)
# --------------------------------------------------------------------------------------------

def test_record_validity():
    L, N = 10, 4
    ok = W.encode(2, [3], [0, 0, 1, W.IDLE])
    assert parse_record(ok, L, N) is not None
    bad = [
        W.encode(0, [], [0, 0, 0, 0]),                  # S = 0
        W.encode(5, [1, 2, 3, 4], [0, 1, 2, 3]),        # S > N
        W.encode(9, [1, 2, 3, 4, 5, 6, 7], [0] * 8),    # S > 8
        W.encode(2, [9], [0, 1, 1, 1]),                 # cut = L-1
        W.encode(3, [4, 4], [0, 1, 2, 2]),              # cuts not increasing
        W.encode(3, [5, 4], [0, 1, 2, 2]),
        W.encode(2, [3], [0, 0, 0, W.IDLE]),            # stage 1 without worker
        W.encode(2, [3], [0, 1, 1, 1, 0]),              # worker 4 >= N has a stage
        W.encode(2, [3], [0, 2, 1, 1]),                 # stage id >= S
        W.encode(2, [3], [0, 0xFE, 1, 1]),
    ]
    for rec in bad:
        assert parse_record(rec, L, N) is None
        assert time_ns(None, None, parse_record(rec, L, N)) == (1 << 64) - 1
    # entries past S-1 are ignored
    rec = bytearray(ok)
    rec[3] = 0
    assert parse_record(bytes(rec), L, N) is not None


def test_switch_bytes():
    prof = W.Profile("s", [0] * 4, [0] * 4, [1, 10, 100, 1000], [1] * 4, [1] * 4)
    a = Partition(2, [1], [[0], [1]])
    assert switch_bytes(prof, a, a) == 0
    b = Partition(2, [2], [[0], [1]])        # layer 2 moves from worker 1 to worker 0
    assert switch_bytes(prof, b, a) == 100
    c = Partition(2, [1], [[0, 2], [1]])     # worker 2 joins stage 0: receives layers 0,1
    assert switch_bytes(prof, c, a) == 11
    d = Partition(1, [], [[3]])              # a fresh worker receives everything
    assert switch_bytes(prof, d, a) == 1111
