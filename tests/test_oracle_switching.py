"""Pins of the switching-cost oracle (oracle/switching.py; reading F-2).

refill: the startup state of Fig. 2 (values the paper prints), a closed form for the ideal pipeline
at every S, a hand-derived two-stage case with communication, and S = 1 (no pipeline, nothing to
refill). migrate: hand-worked moves (one source, the cheaper of two holders, two messages rounded
separately) and the identity sum over workers of gained bytes = switch_bytes, whose definition
(oracle.model.switch_bytes, SPEC §6) is written independently of the message walk.
"""
import os
import pytest

import workloads as W
from oracle.model import Partition, encode_partition, parse_record, switch_bytes, xfer
from oracle.neighbourhood import layer_sets
from oracle.sim import time_ns
from oracle.switching import (gained_messages, migrate_ns, refill_ns, startup_completions,
                              switch_reward, switch_rewards)

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


def uniform(S, f, b, c=0, layers_per_stage=1):
    L = S * layers_per_stage
    prof = W.Profile("u", [c] * L, [c] * L, [0] * L, [f] * L, [b] * L)
    st = W.State([[f] * L for _ in range(S)], [[b] * L for _ in range(S)],
                 [[0 if u == v else 10**6 for v in range(S)] for u in range(S)])
    m = layers_per_stage
    return prof, st, Partition(S, [m * (i + 1) - 1 for i in range(S - 1)], [[s] for s in range(S)])


def test_fig2_startup_state():
    """Fig. 2: completions 12, 15, 18, 21; refill 9."""
    g = _golden("fig2_startup.txt")
    S, f, b = int(g["workers"]), int(g["F"]), int(g["B"])
    prof, st, p = uniform(S, f, b, int(g["comm"]))
    T = time_ns(prof, st, p)
    assert T == int(g["steady_period"])
    assert startup_completions(prof, st, p, S) == [int(x) for x in g["completions"].split()]
    assert refill_ns(prof, st, p, T) == int(g["refill"])


@pytest.mark.parametrize("S", range(1, 9))
@pytest.mark.parametrize("f,b", [(1, 2), (3, 1), (5, 5), (2, 7)])
def test_ideal_pipeline_refill_closed_form(S, f, b):
    """Ideal pipeline (equal stages, no communication): mini-batch 0 takes S f forward plus S b
    backward, then one completes every f + b, so refill = (2S-1)(f+b) - S(f+b) = (S-1)(f+b)."""
    prof, st, p = uniform(S, f, b, layers_per_stage=2)
    T = time_ns(prof, st, p)
    assert T == 2 * (f + b)
    C = startup_completions(prof, st, p, S)
    assert C[0] == S * T
    assert refill_ns(prof, st, p, T) == (S - 1) * T


def test_two_stage_startup_by_hand():
    g = _golden("two_stage_startup.txt")
    f, b, c = [int(x) for x in g["F"].split()], [int(x) for x in g["B"].split()], int(g["comm"])
    prof = W.Profile("h", [c, c], [c, c], [0, 0], f, b)
    st = W.State([f, f], [b, b], [[0, 10**6], [10**6, 0]])
    p = Partition(2, [0], [[0], [1]])
    T = time_ns(prof, st, p)
    assert T == int(g["T"])
    assert startup_completions(prof, st, p, 2) == [int(x) for x in g["completions"].split()]
    assert refill_ns(prof, st, p, T) == int(g["refill"])


def test_single_stage_has_nothing_to_refill():
    """S = 1: no pipeline; the first mini-batch completes after one (F + B), which is T (or less
    than T when the all-reduce of replicas dominates), so refill = 0."""
    prof = W.vgg16()
    for N in (1, 2, 4):
        st = W.make_state(prof, [1 + w for w in range(N)], nic_gbps=[10] * N)
        p = Partition(1, [], [list(range(N))])
        T = time_ns(prof, st, p)
        assert startup_completions(prof, st, p, 1)[0] <= T
        assert refill_ns(prof, st, p, T) == 0


def _mini():
    """4 layers with weights 1000, 2000, 3000, 4001 bytes; 3 workers."""
    prof = W.Profile("m", [10] * 4, [10] * 4, [1000, 2000, 3000, 4001], [5] * 4, [10] * 4)
    st = W.State([[5] * 4] * 3, [[10] * 4] * 3,
                 [[0, 3 * 10**6, 7 * 10**6], [2 * 10**6, 0, 10**6], [5 * 10**5, 10**6, 0]])
    return prof, st


def test_migrate_single_source():
    """Worker 1 newly holds layers 2, 3 (7001 bytes) that only worker 0 held: one message over
    tau[0][1] = 3 ns/B."""
    prof, st = _mini()
    old = Partition(1, [], [[0]])
    new = Partition(2, [1], [[0], [1]])
    assert gained_messages(prof, st, new, old) == [[], [(7001, 21003)], []]
    assert migrate_ns(prof, st, new, old) == 21003


def test_migrate_cheapest_holder_and_separate_messages():
    """Old: layers 0-1 on {0, 1}, layers 2-3 on {2}; new: every layer on {0, 1, 2}.
    Worker 2 gains layers 0-1 (3000 B) from the cheaper holder, 1->2 at 1 ns/B (not 0->2 at 7 ns/B).
    Workers 0 and 1 gain layers 2-3 (7001 B) from worker 2: 0.5 ns/B -> ceil(3500.5) = 3501 and
    1 ns/B -> 7001. Then a worker gaining from two old stages receives two messages, each rounded
    on its own."""
    prof, st = _mini()
    old = Partition(2, [1], [[0, 1], [2]])
    new = Partition(1, [], [[0, 1, 2]])
    msgs = gained_messages(prof, st, new, old)
    assert msgs == [[(7001, 3501)], [(7001, 7001)], [(3000, 3000)]]
    assert migrate_ns(prof, st, new, old) == 7001
    # worker 0 gains layer 0 from {1} (2 ns/B) and layers 1-3 from {2} (0.5 ns/B)
    old2 = Partition(2, [0], [[1], [2]])
    new2 = Partition(1, [], [[0]])
    prof2 = W.Profile("m2", [10] * 4, [10] * 4, [1001, 2000, 3000, 4001], [5] * 4, [10] * 4)
    m = gained_messages(prof2, st, new2, old2)[0]
    assert m == [(1001, xfer(1001, 2 * 10**6)), (9001, xfer(9001, 5 * 10**5))]
    assert m[1][1] == 4501  # ceil(9001 / 2)


def test_gained_bytes_sum_to_switch_bytes():
    """sum_w (bytes of w's messages) = sum_l P[l] |W_new(l) \\ W_old(l)| (SPEC §6), for random
    partitions; with tau = 1 ns/B every message lasts exactly its bytes."""
    prof = W.resnet50()
    L = len(prof.O)
    for N in (2, 5, 8):
        st = W.State([list(prof.f_ref)] * N, [list(prof.b_ref)] * N,
                     [[0 if u == v else 10**6 for v in range(N)] for u in range(N)])
        recs = W.sample_records(L, N, 60, seed=N, random_placement_p=0.7)
        for i in range(0, 60, 2):
            a, b = parse_record(bytes(recs[i]), L, N), parse_record(bytes(recs[i + 1]), L, N)
            msgs = gained_messages(prof, st, a, b)
            assert sum(x for m in msgs for x, _ in m) == switch_bytes(prof, a, b)
            assert all(d == x for m in msgs for x, d in m)
            assert migrate_ns(prof, st, a, b) == max(sum(x for x, _ in m) for m in msgs)


def test_unchanged_partition_costs_nothing():
    """Same layer set on every worker -> no pause, no refill, no migration: reward = T."""
    prof = W.vgg16()
    st = W.vgg_state()
    p = Partition(3, [5, 12], [[0, 1], [2], [3]])
    rec = encode_partition(p)
    T, R, M, Rw = switch_reward(prof, st, rec, p, 10)
    assert (R, M, Rw) == (0, 0, T) and T == time_ns(prof, st, p)
    # a different record with the same per-worker layer sets (stage order is fixed by layers, so
    # only an idle worker staying idle qualifies) is unchanged too
    assert layer_sets(parse_record(rec, len(prof.O), 8), len(prof.O), 8) == layer_sets(p, len(prof.O), 8)


def test_reward_amortises_over_horizon():
    prof = W.vgg16()
    st = W.vgg_state()
    cur = Partition(2, [9], [[0], [1]])
    new = encode_partition(Partition(2, [10], [[0], [1]]))
    T, R, M, r1 = switch_reward(prof, st, new, cur, 1)
    assert R + M > 0 and r1 == T + R + M
    _, _, _, rh = switch_reward(prof, st, new, cur, 10**15)
    assert rh == T + 1
    _, _, _, r7 = switch_reward(prof, st, new, cur, 7)
    assert r7 == T + -(-(R + M) // 7)
    # invalid proposals score UINT64_MAX everywhere; an invalid current partition is an error
    bad = bytes([9] + [0xFF] * 15)
    assert switch_rewards(prof, st, [bad], encode_partition(cur), 3) == [((1 << 64) - 1,) * 4]
    with pytest.raises(ValueError):
        switch_rewards(prof, st, [new], bad, 3)
    with pytest.raises(ValueError):
        switch_rewards(prof, st, [new], encode_partition(cur), 0)
