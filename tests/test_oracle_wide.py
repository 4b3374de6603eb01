"""Pins of the oracle on wide partitions (NEXT row f4: S <= 16 stages and N <= 16 workers in a 32-byte
record, for the paper's 10-GPU testbed), CPU only.

The simulation and the enumeration are written for any S and N; what is new is the 32-byte record
and the sizes. The pins below hold at those sizes for reasons outside the code: the uniform-layer
closed form of the 1F1B period (tests/golden/uniform_closed_form.txt's formula, Observation 3 at
PAPER.md:521-580) at S = 10..16, the serial time at S = 1, pure data parallelism over 10 or 16
replicas (Fig. 1a with a ring all-reduce), the textbook min-max
partition at S up to 12, and the enumeration counted by itertools.
"""
from fractions import Fraction
from itertools import combinations
from math import comb

import numpy as np
import pytest

import workloads as W
from oracle.enumerate import USE_ALL_WORKERS, candidates, count, decode, index_of
from oracle.model import Partition, ceil_div, encode_partition, parse_record, xfer
from oracle.sim import simulate, time_ns


def test_wide_record_rules():
    L, N = 40, 10
    sow = [0, 1, 2, 3, 4, 5, 6, 7, 8, 9] + [0xFF] * 6
    ok = W.encode(10, [3, 7, 11, 15, 19, 23, 27, 31, 35], sow, wide=True)
    p = parse_record(ok, L, N)
    assert p is not None and p.S == 10 and p.W == [[w] for w in range(10)]
    assert p.cuts == [3, 7, 11, 15, 19, 23, 27, 31, 35]
    assert encode_partition(p, wide=True) == ok
    assert parse_record(ok, L, 9) is None                       # worker 9 does not exist (and S > N)
    assert parse_record(W.encode(11, list(range(1, 11)), list(range(11)) + [0xFF] * 5, wide=True), L, N) is None
    assert parse_record(W.encode(17, [], [0] * 16, wide=True), L, 16) is None      # S > 16
    assert parse_record(W.encode(16, list(range(15)), list(range(16)), wide=True), L, 16) is not None
    assert parse_record(W.encode(2, [5, 4], [0, 1] + [0xFF] * 14, wide=True), L, N).cuts == [5]  # S - 1 cuts used
    assert parse_record(W.encode(2, [5], [0, 0] + [0xFF] * 14, wide=True), L, N) is None     # stage 1 empty
    assert parse_record(W.encode(2, [39], [0, 1] + [0xFF] * 14, wide=True), L, N) is None    # cut = L - 1
    assert parse_record(W.encode(2, [5], [0, 2] + [0xFF] * 14, wide=True), L, N) is None     # stage id >= S
    # a 16-byte record keeps its limits (S <= 8, workers < 8) whatever N is
    assert parse_record(W.encode(9, list(range(8)), list(range(8))), L, 16) is None
    with pytest.raises(ValueError):
        parse_record(b"\x01" * 24, L, N)


def uniform_wide(L, S, f, b, c, N=None, fs=10**6):
    N = N or S
    prof = W.Profile("u", [c] * L, [c] * L, [0] * L, [f] * L, [b] * L)
    st = W.State([[f] * L for _ in range(N)], [[b] * L for _ in range(N)],
                 [[0 if u == v else fs for v in range(N)] for u in range(N)])
    m = L // S
    rec = W.contiguous_record(L, [m * (i + 1) - 1 for i in range(S - 1)], [1] * S, wide=True)
    return prof, st, parse_record(rec, L, N)


@pytest.mark.parametrize("L,S,f,b,c", [(20, 10, 3, 6, 5), (24, 12, 2, 4, 7), (32, 16, 1, 2, 0),
                                       (48, 16, 10, 20, 1000), (30, 10, 5, 5, 100), (16, 16, 7, 9, 3)])
def test_uniform_closed_form_wide(L, S, f, b, c):
    """lambda = max(m(f+b), (L(f+b) + 2(S-1)c)/S, c) for uniform layers, now at 10-16 stages."""
    m = L // S
    expect = max(Fraction(m * (f + b)), Fraction(L * (f + b) + 2 * (S - 1) * c, S), Fraction(c))
    assert simulate(*uniform_wide(L, S, f, b, c)) == expect


def test_single_stage_serial_on_a_wide_record():
    rng = np.random.default_rng(31)
    for _ in range(10):
        L = int(rng.integers(1, 12))
        prof = W.random_profile(L, rng)
        st = W.random_state_small(prof, 12, rng)
        w = int(rng.integers(8, 12))                      # a worker a 16-byte record cannot name
        p = parse_record(W.encode(1, [], [0xFF] * w + [0], wide=True), L, 12)
        assert p.W == [[w]]
        assert simulate(prof, st, p) == sum(st.f[w]) + sum(st.b[w])


@pytest.mark.parametrize("r", [10, 16])
def test_data_parallel_many_replicas(r):
    """S = 1 over r homogeneous replicas: lambda = max(ceil(F/r) + ceil(B/r), 2(r-1) ceil(ceil(P/r) tau/1e6))."""
    for F, B, P, tau in [(70, 90, 10**6 + 1, 10**6), (1000, 2000, 10, 10**6), (5, 5, 999_999, 3 * 10**6)]:
        prof = W.Profile("dp", [0], [0], [P], [F], [B])
        st = W.State([[F]] * r, [[B]] * r, [[0 if u == v else tau for v in range(r)] for u in range(r)])
        p = parse_record(W.encode(1, [], [0] * r, wide=True), 1, r)
        expect = max(ceil_div(F, r) + ceil_div(B, r), 2 * (r - 1) * xfer(ceil_div(P, r), tau))
        assert simulate(prof, st, p) == expect


def _minmax_partition(cost, S):
    L = len(cost)
    pre = [0]
    for c in cost:
        pre.append(pre[-1] + c)
    best = {(0, 0): 0}
    for s in range(1, S + 1):
        for e in range(s, L + 1):
            best[(s, e)] = min(max(best[(s - 1, a)], pre[e] - pre[a]) for a in range(s - 1, e) if (s - 1, a) in best)
    return best[(S, L)]


def test_zero_comm_min_max_partition_wide():
    """No communication, identical workers, one per stage: the period is the bottleneck stage, so the
    best S-stage partition (S up to 12) costs the textbook min-max contiguous partition."""
    rng = np.random.default_rng(33)
    for _ in range(4):
        L = int(rng.integers(10, 15))
        S = min(int(rng.integers(9, 13)), L)
        f = [int(x) for x in rng.integers(1, 50, size=L)]
        prof = W.Profile("z", [0] * L, [0] * L, [0] * L, f, [2 * x for x in f])
        st = W.State([f] * S, [[2 * x for x in f]] * S, [[0] * S for _ in range(S)])
        best = min(time_ns(prof, st, Partition(S, list(c), [[s] for s in range(S)]))
                   for c in combinations(range(L - 1), S - 1))
        assert best == _minmax_partition([3 * x for x in f], S)


@pytest.mark.parametrize("flags", [0, USE_ALL_WORKERS])
def test_enumeration_at_ten_workers(flags):
    """The index order of SPEC §5 with N = 10 and S up to 10: sizes by counting, round trips."""
    L, N = 12, 10
    assert count(L, N, 1, 10, flags) == sum(
        (comb(N - 1, S - 1) if flags else comb(N, S)) * comb(L - 1, S - 1) for S in range(1, 11))
    n = 0
    for i, p in enumerate(candidates(L, N, 8, 10, flags)):
        if i % 97 == 0:
            assert index_of(L, N, 8, 10, flags, p) == i
            assert decode(L, N, 8, 10, flags, i) == p
        n += 1
    assert n == count(L, N, 8, 10, flags)
