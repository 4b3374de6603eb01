"""Pins of the oracle's enumeration, brute force, parametric DP and cycle-ratio cross-check (CPU)."""
from itertools import combinations
from math import comb

import numpy as np
import pytest

import workloads as W
from oracle.cycle_ratio import max_cycle_ratio
from oracle.enumerate import (USE_ALL_WORKERS, candidates, count, decode, index_of, lex_rank,
                              lex_unrank)
from oracle.param_dp import optimum
from oracle.search import brute_force
from oracle.sim import simulate


# --------------------------------------------------------------------------------------------
# index order (SPEC §5)
# --------------------------------------------------------------------------------------------

def test_lex_rank_matches_itertools():
    for n in range(0, 9):
        for k in range(0, n + 1):
            for i, c in enumerate(combinations(range(n), k)):
                assert lex_rank(c, n) == i
                assert lex_unrank(i, n, k) == list(c)


@pytest.mark.parametrize("L,N,smin,smax,flags", [(8, 4, 1, 4, 0), (8, 4, 1, 4, 1), (5, 3, 2, 3, 0),
                                                 (6, 5, 1, 5, 1), (3, 6, 1, 3, 0), (1, 2, 1, 2, 0)])
def test_index_roundtrip(L, N, smin, smax, flags):
    seen = 0
    for i, p in enumerate(candidates(L, N, smin, smax, flags)):
        assert index_of(L, N, smin, smax, flags, p) == i
        q = decode(L, N, smin, smax, flags, i)
        assert (q.S, q.cuts, q.W) == (p.S, p.cuts, p.W)
        seen += 1
    assert seen == count(L, N, smin, smax, flags)


def test_config_space_sizes():
    """toy 165 (120 with sum r = N); VGG 1,184,040; GPT-96 S=8: C(95,7)."""
    assert count(8, 4, 1, 4) == 165
    assert count(8, 4, 1, 4, USE_ALL_WORKERS) == 120
    assert count(21, 8, 1, 8) == 1_184_040
    assert count(96, 8, 8, 8) == comb(95, 7) == 11_050_084_695
    assert count(96, 8, 1, 8) == 19_813_501_785
    assert count(18, 8, 1, 8) == 480_700
    assert count(26, 8, 1, 8) == 4_272_048


def test_contiguous_placement():
    """Reading C-11: stage s gets workers [R_{s-1}, R_s)."""
    p = decode(10, 6, 3, 3, 0, 0)
    assert p.W == [[0], [1], [2]] and p.cuts == [0, 1]
    last = decode(10, 6, 3, 3, 0, count(10, 6, 3, 3) - 1)
    assert last.W == [[0, 1, 2, 3], [4], [5]] and last.cuts == [7, 8]


# --------------------------------------------------------------------------------------------
# search pins: brute force over tiny spaces == parametric DP (value AND lexicographic-first index)
# --------------------------------------------------------------------------------------------

def test_toy_brute_force_equals_dp():
    prof, st = W.toy(), W.toy_state()
    T, idx, part, n = brute_force(prof, st, 1, 4)
    assert n == 165
    T2, idx2, _ = optimum(prof, st, 1, 4)
    assert (T, idx) == (T2, idx2)


def test_random_brute_force_equals_dp():
    rng = np.random.default_rng(21)
    done = 0
    while done < 80:
        L = int(rng.integers(1, 8))
        N = int(rng.integers(1, 5))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([20, 1000])),
                                bytes_max=int(rng.choice([100, 5000])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([100, 3000])))
        flags = int(rng.integers(0, 2))
        smax = min(N, L, 4)
        smin = int(rng.integers(1, smax + 1))
        T, idx, _, n = brute_force(prof, st, smin, smax, flags)
        if n == 0:
            continue
        assert optimum(prof, st, smin, smax, flags)[:2] == (T, idx)
        done += 1


def test_dp_ties_take_lowest_index():
    """All-equal layers and free links create many ties; the first index must win (C-13)."""
    L, N = 6, 3
    prof = W.Profile("tie", [0] * L, [0] * L, [0] * L, [2] * L, [2] * L)
    st = W.State([[2] * L] * N, [[2] * L] * N, [[0] * N for _ in range(N)])
    T, idx, _, _ = brute_force(prof, st, 1, 3)
    assert optimum(prof, st, 1, 3)[:2] == (T, idx)


# --------------------------------------------------------------------------------------------
# the simulation equals the max cycle ratio of the explicit event graph (independent method)
# --------------------------------------------------------------------------------------------

def test_simulation_equals_max_cycle_ratio():
    rng = np.random.default_rng(31)
    n = 0
    for it in range(40):
        L = int(rng.integers(1, 6))
        N = int(rng.integers(1, 6))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([10, 1000])),
                                bytes_max=int(rng.choice([10, 4000])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([10, 3000])))
        from oracle.model import parse_record
        for r in W.sample_records(L, N, 8, 1000 + it, s_max=3):
            p = parse_record(bytes(r), L, N)
            if p is None or sum(len(w) for w in p.W) > 5:
                continue
            assert simulate(prof, st, p) == max_cycle_ratio(prof, st, p)
            n += 1
    assert n > 150


def test_toy_all_candidates_cycle_ratio():
    prof, st = W.toy(), W.toy_state()
    for p in candidates(8, 4, 1, 3):
        assert simulate(prof, st, p) == max_cycle_ratio(prof, st, p)


def test_ceil_cycle_ratio_equals_simulation():
    """The long-transient fallback of time_ns (Bellman-Ford on the event graph) equals ceil(lambda)
    of the simulation wherever the simulation finishes."""
    from oracle.cycle_ratio import ceil_max_cycle_ratio
    from oracle.model import parse_record
    rng = np.random.default_rng(41)
    n = 0
    for it in range(30):
        L = int(rng.integers(1, 12))
        N = int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([10, 10**6])), bytes_max=int(rng.choice([10, 10**7])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([10, 10**5])))
        for r in W.sample_records(L, N, 10, 2000 + it):
            p = parse_record(bytes(r), L, N)
            if p is None:
                continue
            lam = simulate(prof, st, p)
            assert ceil_max_cycle_ratio(prof, st, p) == -(-lam.numerator // lam.denominator)
            n += 1
    assert n > 200


def test_long_transient_uses_cycle_ratio():
    """A GNMT-16 partition (trace state 11) whose bottleneck worker cycle (207,874,737 ns) beats another
    stage's (207,821,004 ns) by 0.03%: the faster stage takes thousands of rounds to lock in. time_ns
    does not wait (cap TIME_NS_ROUNDS) and takes ceil(lambda) from the event graph; the full
    simulation, given enough rounds, agrees."""
    from oracle.model import Partition
    from oracle.sim import NoPeriod, time_ns
    prof = W.profile("gnmt16")
    st = W.trace_c3(prof)[-1]
    part = Partition(5, [6, 8, 11, 15], [[0], [1], [2], [3], [4]])
    with pytest.raises(NoPeriod):
        simulate(prof, st, part, max_rounds=2000)
    lam = simulate(prof, st, part, max_rounds=100_000)
    assert lam == 207_874_737
    assert time_ns(prof, st, part) == 207_874_737


# --------------------------------------------------------------------------------------------
# the two-worker neighbourhood, by definition
# --------------------------------------------------------------------------------------------

def test_neighbourhood_by_hand():
    """L = 3 layers, N = 2 workers, p = stage [0] on w0, stage [1,2] on w1. With two workers every
    other valid partition differs in at most two entries of the per-worker layer array, so the
    neighbourhood is all six others (derived by hand in oracle/neighbourhood.py's docstring terms)."""
    from oracle.model import Partition, encode_partition
    from oracle.neighbourhood import all_partitions, neighbourhood
    p = Partition(2, [0], [[0], [1]])
    want = sorted([
        W.encode(1, [], [0, 0]), W.encode(1, [], [0, W.IDLE]), W.encode(1, [], [W.IDLE, 0]),
        W.encode(2, [0], [1, 0]), W.encode(2, [1], [0, 1]), W.encode(2, [1], [1, 0]),
    ])
    assert neighbourhood(3, 2, p) == want
    assert len(list(all_partitions(3, 2))) == 7


def test_neighbourhood_distance_one_moves():
    """L = 2, N = 3, p = one stage on w0 (w1, w2 idle). Single-worker changes: w1 or w2 joins the
    stage (w0 cannot change alone: the layers would be uncovered)."""
    from oracle.model import Partition, encode_partition
    from oracle.neighbourhood import layer_sets, neighbourhood
    p = Partition(1, [], [[0]])
    nb = neighbourhood(2, 3, p)
    from oracle.model import parse_record
    d1 = [r for r in nb if sum(a != b for a, b in zip(layer_sets(parse_record(r, 2, 3), 2, 3),
                                                       layer_sets(p, 2, 3))) == 1]
    assert sorted(d1) == sorted([W.encode(1, [], [0, 0, W.IDLE]), W.encode(1, [], [0, W.IDLE, 0])])


def test_neighbourhood_symmetric():
    from oracle.model import parse_record
    from oracle.neighbourhood import all_partitions, neighbourhood
    from oracle.model import encode_partition
    L, N = 4, 3
    parts = list(all_partitions(L, N))
    nbs = {encode_partition(p): set(neighbourhood(L, N, p)) for p in parts[::3]}
    for a, na in nbs.items():
        for b in na:
            if b in nbs:
                assert a in nbs[b]
