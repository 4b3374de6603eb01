"""Pins of the round-robin replica oracle (NEXT row f4, reading F-5; oracle/roundrobin.py):

* every r_s = 1: the round-robin schedule is the static 1F1B of reading C-2, so lambda equals
  oracle.sim's (an independent simulator of the same schedule), exactly;
* S = 1: replica i runs F, B, F, B, ... on every r-th mini-batch: lambda = max_i (F_i + B_i) / r
  (identical replicas: (F + B) / r, PipeDream's data parallelism);
* a hand-derived two-stage case (tests/golden/roundrobin_two_stage.txt);
* the simulation equals the maximum cycle ratio of the explicit timed event graph of one period
  (Johnson's elementary cycles over the lcm(r)-unrolled graph), on tiny random instances;
* invariants: lambda >= every replica's (F + B) / r_s, every link's transfer / lcm(r_s, r_{s+1}),
  every sync term d_s / r_s; monotone in the durations.
"""
import os
from fractions import Fraction

import numpy as np
import pytest

import workloads as W
from oracle import roundrobin as RR
from oracle import sim
from oracle.model import Partition, ceil_div

HERE = os.path.dirname(os.path.abspath(__file__))


def _random_partition(rng, L, N, S, max_r=3):
    cuts = sorted(int(x) for x in rng.choice(L - 1, S - 1, replace=False)) if S > 1 else []
    sizes = [1] * S
    left = N - S
    for s in range(S):
        add = int(rng.integers(0, min(max_r - 1, left) + 1)) if left > 0 else 0
        sizes[s] += add
        left -= add
    perm = [int(x) for x in rng.permutation(N)]
    W_, o = [], 0
    for r in sizes:
        W_.append(sorted(perm[o:o + r]))
        o += r
    return Partition(S, cuts, W_)


@pytest.mark.parametrize("seed", range(6))
def test_r1_equals_split_model(seed):
    rng = np.random.default_rng(700 + seed)
    for _ in range(6):
        L = int(rng.integers(2, 10))
        N = int(rng.integers(1, 7))
        S = int(rng.integers(1, min(N, L) + 1))
        prof = W.random_profile(L, rng, f_max=900, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        cuts = sorted(int(x) for x in rng.choice(L - 1, S - 1, replace=False)) if S > 1 else []
        ws = [int(x) for x in rng.permutation(N)[:S]]
        part = Partition(S, cuts, [[w] for w in ws])
        assert RR.rr_lambda(prof, st, part) == sim.simulate(prof, st, part)
        assert RR.time_ns(prof, st, part) == sim.time_ns(prof, st, part)


@pytest.mark.parametrize("r", [1, 2, 3, 5, 8])
def test_single_stage_data_parallel(r):
    L = 4
    prof = W.Profile("dp", [10] * L, [10] * L, [0] * L, [3] * L, [5] * L)
    st = W.State([[3] * L] * r, [[5] * L] * r, [[0 if u == v else 100 for v in range(r)] for u in range(r)])
    part = Partition(1, [], [list(range(r))])
    assert RR.rr_lambda(prof, st, part) == Fraction(4 * (3 + 5), r)   # weights 0: no sync term
    # heterogeneous replicas: the slowest one bounds the stage
    rng = np.random.default_rng(r)
    f = [[int(x) for x in rng.integers(1, 50, L)] for _ in range(r)]
    b = [[int(x) for x in rng.integers(1, 90, L)] for _ in range(r)]
    st2 = W.State(f, b, st.tau)
    want = max(Fraction(sum(f[w]) + sum(b[w]), r) for w in range(r))
    assert RR.rr_lambda(prof, st2, part) == want


def test_two_stage_golden():
    """tests/golden/roundrobin_two_stage.txt: stage 0 on two identical replicas (F = 2, B = 4 whole
    mini-batch), stage 1 on one worker (F = 1, B = 2), free links. Each replica takes every other
    mini-batch and keeps m_0 = ceil(3 / 2) = 2 of its own in flight: stage 0 finishes one mini-batch
    per (2 + 4) / 2 = 3, stage 1 one per 1 + 2 = 3, the loop through both stages carries 4 mini-batches
    for 2 + 1 + 2 + 4 = 9: lambda = 3. With a forward transfer of 8 on both links the links carry
    one mini-batch each per 2 (8 / 2 = 4) and the loop 2 + 8 + 1 + 2 + 4 = 17 per 4 mini-batches:
    lambda = 17 / 4, T = 5."""
    rows = {}
    with open(os.path.join(HERE, "golden", "roundrobin_two_stage.txt")) as fh:
        for line in fh:
            line = line.strip()
            if line and not line.startswith("#"):
                k, v = line.split("=")
                rows[k.strip()] = Fraction(v.strip())
    prof = W.Profile("g", [1, 0], [0, 1], [0, 0], [0, 0], [0, 0])
    tau0 = [[0, 0, 0], [0, 0, 0], [0, 0, 0]]
    st = W.State([[2, 0], [2, 0], [0, 1]], [[4, 0], [4, 0], [0, 2]], tau0)
    part = Partition(2, [0], [[0, 1], [2]])
    assert RR.rr_lambda(prof, st, part) == rows["lambda_free_links"]
    tau = [[0, 0, 8 * 10**6], [0, 0, 8 * 10**6], [0, 0, 0]]   # O[0] = 1 byte -> 8 ns forward
    st2 = W.State(st.f, st.b, tau)
    lam = RR.rr_lambda(prof, st2, part)
    assert lam == rows["lambda_forward_8"]
    assert RR.time_ns(prof, st2, part) == ceil_div(lam.numerator, lam.denominator) == 5
    assert RR.max_cycle_ratio(prof, st2, part) == lam


@pytest.mark.parametrize("seed", range(8))
def test_simulation_equals_cycle_ratio(seed):
    rng = np.random.default_rng(900 + seed)
    for _ in range(3):
        L = int(rng.integers(2, 6))
        N = int(rng.integers(2, 6))
        S = int(rng.integers(1, min(3, N, L) + 1))
        prof = W.random_profile(L, rng, f_max=500, bytes_max=10**4)
        st = W.random_state_small(prof, N, rng, tau_max=2000)
        part = _random_partition(rng, L, N, S)
        ing = RR.RRIngredients(prof, st, part)
        assert RR.compute_lambda(ing) == RR.max_cycle_ratio(prof, st, part), (part, ing.r)


@pytest.mark.parametrize("seed", range(4))
def test_bounds_and_monotonicity(seed):
    rng = np.random.default_rng(950 + seed)
    for _ in range(5):
        L = int(rng.integers(2, 9))
        N = int(rng.integers(2, 9))
        S = int(rng.integers(1, min(5, N, L) + 1))
        prof = W.random_profile(L, rng, f_max=800, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        part = _random_partition(rng, L, N, S, max_r=4)
        ing = RR.RRIngredients(prof, st, part)
        lam = RR.rr_lambda(prof, st, part)
        for s in range(S):
            r = ing.r[s]
            for w in ing.W[s]:
                assert lam >= Fraction(ing.Fd[s][w] + ing.Bd[s][w], r)
            if r >= 2:
                assert lam >= Fraction(ing.sync[s], r)
        for s in range(S - 1):
            step = RR.lcm(ing.r[s], ing.r[s + 1])
            for k in range(step):
                assert lam >= Fraction(ing.fwd_time(s, k), step)
                assert lam >= Fraction(ing.bwd_time(s, k), step)
        # slower workers never speed the pipeline up
        st2 = W.State([[x * 2 for x in row] for row in st.f], st.b, st.tau)
        assert RR.rr_lambda(prof, st2, part) >= lam


@pytest.mark.parametrize("seed", range(4))
def test_bellman_ford_ceiling_equals_simulation(seed):
    """The fallback for long transients (ceil_lambda_compute: Bellman-Ford on integer theta over the
    one-period event graph) equals ceil of the simulated lambda wherever the simulation settles."""
    rng = np.random.default_rng(980 + seed)
    for _ in range(10):
        L = int(rng.integers(2, 8))
        N = int(rng.integers(2, 7))
        S = int(rng.integers(1, min(4, N, L) + 1))
        prof = W.random_profile(L, rng, f_max=500, bytes_max=10**4)
        st = W.random_state_small(prof, N, rng, tau_max=2000)
        part = _random_partition(rng, L, N, S)
        ing = RR.RRIngredients(prof, st, part)
        lam = RR.compute_lambda(ing)
        assert RR.ceil_lambda_compute(ing) == ceil_div(lam.numerator, lam.denominator)


def test_long_transient_uses_the_event_graph():
    """A C5 record (ResNet-50, rollout state 0) with no periodic regime within 20,000 rounds: the
    simulation gives up and ceil(lambda) comes from the event graph."""
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    part = Partition(3, [15, 29], [[4], [0, 3], [2]])
    ing = RR.RRIngredients(prof, st, part)
    with pytest.raises(RR.NoPeriod):
        RR.compute_lambda(ing, RR.TIME_NS_ROUNDS)
    assert RR.time_ns(prof, st, part) == RR.ceil_lambda_compute(ing) == 591221519
