"""Pins of the schedule-variant oracle (NEXT row f3, oracle/schedules.py; reading F-3), CPU only.

What fixes each mode independently of the code under test:
* GPipe: a hand-worked timeline (tests/golden/flush_two_stage.txt); for one worker
  per stage the forward and the backward phase are permutation flow shops of M identical jobs whose
  machines are the stages and links, so the makespan is the textbook sum(p) + (M - 1) max(p) per
  phase; uniform stages without communication give (M + S - 1)(f + b) (GPipe's bubble, S - 1 slots);
  recompute makes every backward op F' + B'.
* DAPPLE / 1F1B with flush: the hand-worked timeline; the same (M + S - 1)(f + b)
  for uniform stages (1F1B-with-flush has GPipe's bubble); M = 1 is one micro-batch down and up the
  pipeline (the serial chain); S = 1 is M back-to-back micro-batches per replica.
* both flushed schedules: the longest path of the explicit event DAG (an independent formulation)
  on random tiny instances with replicas, PS and ring.
* PS: hand cases; with uniform links and r | P it moves what a ring all-reduce
  moves (2(r - 1) chunks of P / r per worker), so it equals the ring time.
* 2BW: M = 1 is PipeDream; the compute part is M x the 1F1B period (the uniform
  closed form of tests/golden/uniform_closed_form.txt); pure data parallelism gives
  max(M (ceil(F/2) + ceil(B/2)), sync) in both regimes.
"""
import os
from fractions import Fraction

import numpy as np
import pytest

import workloads as W
from oracle import schedules as SC
from oracle.model import Partition, ceil_div, ingredients, xfer
from oracle.sim import simulate, time_ns

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    out = {}
    with open(os.path.join(GOLD, name)) as fh:
        for line in fh:
            line = line.strip()
            if line and not line.startswith("#"):
                k, v = line.split(None, 1)
                out[k] = v
    return out


def uniform(L, S, f, b, c, N=None, fs=10**6):
    """L identical layers, one worker per stage, even split; every boundary transfer lasts c ns."""
    N = N or S
    prof = W.Profile("u", [c] * L, [c] * L, [0] * L, [f] * L, [b] * L)
    st = W.State([[f] * L for _ in range(N)], [[b] * L for _ in range(N)],
                 [[0 if u == v else fs for v in range(N)] for u in range(N)])
    m = L // S
    return prof, st, Partition(S, [m * (i + 1) - 1 for i in range(S - 1)], [[s] for s in range(S)])


def hand_two_stage():
    g = _golden("flush_two_stage.txt")
    F, B = list(map(int, g["F"].split())), list(map(int, g["B"].split()))
    cf, cb = int(g["cf"]), int(g["cb"])
    # tau = 1e6 fs/B: one byte per ns; O[0] = cf bytes forward, G[1] = cb bytes backward
    prof = W.Profile("hand", [cf, 0], [0, cb], [0, 0], F, B)
    st = W.State([F, F], [B, B], [[0, 10**6], [10**6, 0]])
    return g, prof, st, Partition(2, [0], [[0], [1]])


def random_r1(rng, L, S, N):
    prof = W.random_profile(L, rng, f_max=500, bytes_max=10**5)
    st = W.random_state_small(prof, N, rng, tau_max=5000)
    cuts = sorted(rng.choice(np.arange(L - 1), size=S - 1, replace=False).tolist())
    ws = rng.permutation(N)[:S].tolist()
    return prof, st, Partition(S, cuts, [[w] for w in ws])


def random_part(rng, L, N):
    S = int(rng.integers(1, min(N, L) + 1))
    cuts = sorted(rng.choice(np.arange(L - 1), size=S - 1, replace=False).tolist())
    perm = rng.permutation(N).tolist()
    k = int(rng.integers(S, N + 1))
    W_ = [[] for _ in range(S)]
    for i, w in enumerate(perm[:k]):
        W_[i if i < S else int(rng.integers(0, S))].append(w)
    return Partition(S, cuts, [sorted(x) for x in W_])


# --------------------------------------------------------------------------------------------
# hand-worked timelines
# --------------------------------------------------------------------------------------------

def test_hand_two_stage_timelines():
    g, prof, st, p = hand_two_stage()
    M = int(g["M"])
    assert SC.flush_makespan(prof, st, p, SC.GPIPE, M) == int(g["gpipe"])
    assert SC.flush_makespan(prof, st, p, SC.GPIPE, M, recompute=True) == int(g["gpipe_recompute"])
    assert SC.flush_makespan(prof, st, p, SC.DAPPLE, M) == int(g["dapple"])
    end, _ = SC.flush_events(prof, st, p, SC.GPIPE, M, False, SC.RING)
    starts = [end[("B", 1, 1, k)] - 6 for k in range(M)]
    assert starts == list(map(int, g["gpipe_w1_B_starts"].split()))
    end, _ = SC.flush_events(prof, st, p, SC.DAPPLE, M, False, SC.RING)
    starts = [end[("B", 0, 0, k)] - 4 for k in range(M)]
    assert starts == list(map(int, g["dapple_w0_B_starts"].split()))


def test_op_lists():
    """GPipe: all forwards then all backwards; DAPPLE: n_s = min(S - s, M) warm-up forwards, then
    1F1B, then the cool-down backwards (the static 1F1B order of sim with a flush)."""
    assert SC.op_list(SC.GPIPE, 3, 1, 2) == [("F", 0), ("F", 1), ("B", 0), ("B", 1)]
    assert SC.op_list(SC.DAPPLE, 3, 0, 4) == [("F", 0), ("F", 1), ("F", 2), ("B", 0), ("F", 3),
                                              ("B", 1), ("B", 2), ("B", 3)]
    assert SC.op_list(SC.DAPPLE, 3, 2, 2) == [("F", 0), ("B", 0), ("F", 1), ("B", 1)]
    assert SC.op_list(SC.DAPPLE, 4, 0, 2) == [("F", 0), ("F", 1), ("B", 0), ("B", 1)]


# --------------------------------------------------------------------------------------------
# closed forms
# --------------------------------------------------------------------------------------------

@pytest.mark.parametrize("S", [1, 2, 3, 5, 8])
def test_uniform_bubble(S):
    """Uniform stages, no communication: (M + S - 1)(f + b) for GPipe and for 1F1B with flush."""
    for M in (1, 2, S, 2 * S + 1):
        for f, b in ((1, 2), (3, 5), (7, 7)):
            prof, st, p = uniform(S, S, f, b, 0)
            expect = (M + S - 1) * (f + b)
            assert SC.flush_makespan(prof, st, p, SC.GPIPE, M) == expect
            assert SC.flush_makespan(prof, st, p, SC.DAPPLE, M) == expect
            assert SC.model_time_ns(prof, st, p, SC.GPIPE, SC.RING, M, True) == (M + S - 1) * (2 * f + b)


def test_gpipe_flow_shop_r1():
    """One worker per stage, heterogeneous stages and links: each phase is a permutation flow shop of
    M identical jobs on machines stage 0, link 0, stage 1, ..., so its makespan is
    sum(p) + (M - 1) max(p); the backward phase starts when the last stage finishes its forwards."""
    rng = np.random.default_rng(11)
    for _ in range(40):
        L, N = int(rng.integers(2, 12)), int(rng.integers(1, 6))
        S = int(rng.integers(1, min(L, N) + 1))
        prof, st, p = random_r1(rng, L, S, N)
        ing = ingredients(prof, st, p)
        Fs = [ing.Fd[s][p.W[s][0]] for s in range(S)]
        Bs = [ing.Bd[s][p.W[s][0]] for s in range(S)]
        cf = [sum(d for _, _, d in ing.fwd[s]) for s in range(S - 1)]
        cb = [sum(d for _, _, d in ing.bwd[s]) for s in range(S - 1)]
        for M in (1, 2, 5):
            for rc in (False, True):
                Bx = [Bs[s] + (Fs[s] if rc else 0) for s in range(S)]
                fwd = sum(Fs) + sum(cf) + (M - 1) * max(Fs + cf)
                bwd = sum(Bx) + sum(cb) + (M - 1) * max(Bx + cb)
                assert SC.flush_makespan(prof, st, p, SC.GPIPE, M, rc) == fwd + bwd


def test_single_micro_batch_is_serial_chain():
    """M = 1: one micro-batch goes down and back up the pipeline; nothing overlaps."""
    rng = np.random.default_rng(12)
    for _ in range(30):
        L, N = int(rng.integers(2, 10)), int(rng.integers(1, 6))
        S = int(rng.integers(1, min(L, N) + 1))
        prof, st, p = random_r1(rng, L, S, N)
        ing = ingredients(prof, st, p)
        chain = sum(ing.Fd[s][p.W[s][0]] + ing.Bd[s][p.W[s][0]] for s in range(S))
        chain += sum(d for s in range(S - 1) for _, _, d in ing.fwd[s] + ing.bwd[s])
        assert SC.flush_makespan(prof, st, p, SC.GPIPE, 1) == chain
        assert SC.flush_makespan(prof, st, p, SC.DAPPLE, 1) == chain


def test_single_stage_replicas():
    """S = 1 with r replicas: each replica runs M (F + B) back to back; then the synchronisation."""
    prof = W.Profile("dp", [0, 0], [0, 0], [1000, 2001], [3, 4], [5, 6])
    st = W.State([[3, 4], [6, 8], [1, 1]], [[5, 6], [10, 12], [1, 1]],
                 [[0, 10**6, 2 * 10**6], [10**6, 0, 10**6], [3 * 10**6, 10**6, 0]])
    p = Partition(1, [], [[0, 1, 2]])
    ing = ingredients(prof, st, p)
    for M in (1, 3):
        for sched in (SC.GPIPE, SC.DAPPLE):
            for sync in (SC.RING, SC.PS):
                sy = ing.ar[0] if sync == SC.RING else SC.ps_duration(prof.P, 0, 1, [0, 1, 2], st.tau)
                # worker 1: ceil(14/3) + ceil(22/3) = 13 per micro-batch
                assert SC.flush_makespan(prof, st, p, sched, M, False, sync) == 13 * M + sy


# --------------------------------------------------------------------------------------------
# the event DAG (independent formulation)
# --------------------------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(4))
def test_flush_matches_event_dag(seed):
    rng = np.random.default_rng(100 + seed)
    for _ in range(12):
        L, N = int(rng.integers(2, 9)), int(rng.integers(1, 6))
        prof = W.random_profile(L, rng, f_max=300, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        p = random_part(rng, L, N)
        M = int(rng.integers(1, 6))
        for sched in (SC.GPIPE, SC.DAPPLE):
            for sync in (SC.RING, SC.PS):
                rc = bool(rng.integers(0, 2)) and sched == SC.GPIPE
                assert (SC.flush_makespan(prof, st, p, sched, M, rc, sync)
                        == SC.flush_makespan_dag(prof, st, p, sched, M, rc, sync))


# --------------------------------------------------------------------------------------------
# parameter server
# --------------------------------------------------------------------------------------------

def test_ps_hand_cases():
    P = [4, 6]                                     # 10 bytes, shards [0,5) and [5,10) for r = 2
    tau = [[0, 10**6, 0], [3 * 10**6, 0, 0], [0, 0, 0]]
    # push: server 0 gets 5 B from 1 (tau 3e6 -> 15 ns), server 1 gets 5 B from 0 (5 ns): 15
    # pull: server 0 sends 5 B to 1 (5 ns), server 1 sends 5 B to 0 (15 ns): 15
    assert SC.ps_duration(P, 0, 1, [0, 1], tau) == 30
    # r = 3, P = 10: shards 3, 3, 4 bytes; uniform tau 1e6: push = max over servers of 2 x shard = 8
    tau3 = [[0 if u == v else 10**6 for v in range(3)] for u in range(3)]
    assert SC.ps_duration(P, 0, 1, [0, 1, 2], tau3) == 16
    # a replica-free stage synchronises nothing; only the stage's own layers count
    assert SC.ps_duration(P, 0, 1, [2], tau3) == 0
    assert SC.ps_duration(P, 1, 1, [0, 1], tau) == 2 * 9   # 6 bytes: shards 3, 3 at 3e6 fs/B


def test_ps_equals_ring_on_uniform_links():
    """Sharded PS and ring all-reduce both move 2(r - 1) chunks of P / r per worker: equal times when
    every link is the same and r divides P."""
    for r in range(2, 9):
        for Pb, fs in ((r * 1000, 10**6), (r * 7, 3 * 10**6 + 1), (r * 123457, 80_000)):
            tau = [[0 if u == v else fs for v in range(8)] for u in range(8)]
            ws = list(range(r))
            ring = 2 * (r - 1) * xfer(Pb // r, fs)
            assert SC.ps_duration([Pb], 0, 0, ws, tau) == ring


def test_pipedream_with_ps_data_parallel():
    """S = 1, r = 2 under PS: lambda = max(ceil(F/2) + ceil(B/2), PS) (Fig. 1a with a PS)."""
    for F, B, Pb, t01, t10 in [(7, 9, 1001, 10**6, 2 * 10**6), (100, 200, 10, 10**6, 10**6),
                               (10, 11, 10**9, 800_000, 80_000)]:
        prof = W.Profile("dp", [0], [0], [Pb], [F], [B])
        st = W.State([[F], [F]], [[B], [B]], [[0, t01], [t10, 0]])
        p = Partition(1, [], [[0, 1]])
        lo, hi = Pb // 2, Pb - Pb // 2
        ps = max(xfer(lo, t10), xfer(hi, t01)) + max(xfer(lo, t01), xfer(hi, t10))
        expect = max(ceil_div(F, 2) + ceil_div(B, 2), ps)
        assert SC.model_time_ns(prof, st, p, SC.PIPEDREAM, SC.PS) == expect


# --------------------------------------------------------------------------------------------
# 2BW
# --------------------------------------------------------------------------------------------

@pytest.mark.parametrize("row", [l.split() for l in open(os.path.join(GOLD, "uniform_closed_form.txt"))
                                 if l.strip() and not l.startswith("#")])
def test_two_bw_uniform(row):
    """No replicas: one iteration is M periods of the 1F1B steady state, T = ceil(M lambda)."""
    L, S, f, b, c = map(int, row[:5])
    lam = Fraction(row[5])
    prof, st, p = uniform(L, S, f, b, c)
    for M in (1, 2, 3, 7):
        assert SC.model_time_ns(prof, st, p, SC.TWO_BW, SC.RING, M) == ceil_div(
            lam.numerator * M, lam.denominator)


def test_two_bw_data_parallel_regimes():
    """S = 1, r = 2: the synchronisation runs once per M micro-batches, so
    T = max(M (ceil(F/2) + ceil(B/2)), sync) — compute-bound and sync-bound cases."""
    F, B = 7, 9                                   # X = 4 + 5 = 9 per micro-batch
    for Pb, M in ((1000, 1), (1000, 4), (100, 4), (10**5, 4), (10**5, 64)):
        prof = W.Profile("dp", [0], [0], [Pb], [F], [B])
        st = W.State([[F], [F]], [[B], [B]], [[0, 10**6], [10**6, 0]])
        p = Partition(1, [], [[0, 1]])
        ring = 2 * xfer(ceil_div(Pb, 2), 10**6)
        assert SC.model_time_ns(prof, st, p, SC.TWO_BW, SC.RING, M) == max(9 * M, ring)


def test_two_bw_one_micro_batch_is_pipedream():
    rng = np.random.default_rng(13)
    for _ in range(25):
        L, N = int(rng.integers(2, 10)), int(rng.integers(1, 6))
        prof = W.random_profile(L, rng, f_max=300, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        p = random_part(rng, L, N)
        for sync in (SC.RING, SC.PS):
            assert (SC.model_time_ns(prof, st, p, SC.TWO_BW, sync, 1)
                    == SC.model_time_ns(prof, st, p, SC.PIPEDREAM, sync))
        assert SC.model_time_ns(prof, st, p, SC.PIPEDREAM, SC.RING) == time_ns(prof, st, p)


def test_two_bw_pipeline_with_replicas():
    """A replicated pipeline stage: the coalesced chain is the max of M x the compute period (the
    steady state of sim, where nothing waits for the synchronisation) and the sync time."""
    rng = np.random.default_rng(14)
    for _ in range(20):
        L, N = int(rng.integers(3, 10)), int(rng.integers(3, 7))
        prof = W.random_profile(L, rng, f_max=300, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        p = random_part(rng, L, N)
        ing = ingredients(prof, st, p)
        # the compute period: the 1F1B steady state with the all-reduce removed
        ing0 = ingredients(prof, st, p)
        ing0.ar = [0] * p.S
        lam_c = simulate(prof, st, p, ing=ing0)
        for M in (1, 3, 8):
            expect = max([lam_c * M] + [Fraction(ing.ar[s]) for s in range(p.S) if len(p.W[s]) >= 2])
            assert SC.model_time_ns(prof, st, p, SC.TWO_BW, SC.RING, M) == ceil_div(
                expect.numerator, expect.denominator)


def test_two_bw_cycle_route_equals_simulation():
    """The fallback for long transients (max cycle ratio with durations scaled by M, then the sync
    rate) equals the simulation wherever the simulation settles, with and without replicas."""
    rng = np.random.default_rng(16)
    for _ in range(25):
        L, N = int(rng.integers(2, 9)), int(rng.integers(1, 6))
        prof = W.random_profile(L, rng, f_max=300, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        p = random_part(rng, L, N)
        for M in (1, 2, 5):
            for sync in (SC.RING, SC.PS):
                lam = SC.two_bw_lambda(prof, st, p, M, sync)
                assert SC.two_bw_time_ns_cycles(prof, st, p, M, sync) == ceil_div(lam.numerator, lam.denominator)


def test_two_bw_long_transient_state():
    """GNMT-16 states whose 1F1B transients outlast the simulation budget (R-2) still get
    T = max(ceil(M lambda_c), d): between M (ceil(lambda_c) - 1) and M ceil(lambda_c), or the sync d."""
    from oracle.model import parse_record
    prof = W.gnmt16()
    st = W.random_state(prof, 8, np.random.default_rng(17), free_link_p=0.1)
    recs = W.sample_records(prof.L, 8, 150, 41, random_placement_p=0.6)
    for rec in recs:
        p = parse_record(bytes(rec), prof.L, 8)
        if p is None:
            continue
        assert SC.model_time_ns(prof, st, p, SC.TWO_BW, SC.PS, 1) == SC.model_time_ns(prof, st, p, SC.PIPEDREAM, SC.PS)
        ing = SC.model_ingredients(prof, st, p, SC.PS)
        d = max([ing.ar[s] for s in range(p.S) if len(p.W[s]) >= 2] + [0])
        ing.ar = [0] * p.S
        c1 = time_ns(prof, st, p, ing)               # ceil(lambda_compute)
        T8 = SC.model_time_ns(prof, st, p, SC.TWO_BW, SC.PS, 8)
        assert d <= T8 <= max(8 * c1, d)
        assert T8 == d or T8 > 8 * (c1 - 1)


# --------------------------------------------------------------------------------------------
# invariants
# --------------------------------------------------------------------------------------------

def test_flush_invariants():
    """Lower bounds (every worker's own work; the one-micro-batch chain) and strictly increasing in M."""
    rng = np.random.default_rng(15)
    for _ in range(25):
        L, N = int(rng.integers(2, 10)), int(rng.integers(1, 6))
        prof = W.random_profile(L, rng, f_max=300, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        p = random_part(rng, L, N)
        ing = ingredients(prof, st, p)
        work = max(ing.Fd[s][w] + ing.Bd[s][w] for s in range(p.S) for w in p.W[s])
        for sched in (SC.GPIPE, SC.DAPPLE):
            prev = 0
            for M in (1, 2, 4, 7):
                T = SC.flush_makespan(prof, st, p, sched, M)
                assert T >= M * work
                assert T >= SC.flush_makespan(prof, st, p, sched, 1)
                assert T > prev
                prev = T
