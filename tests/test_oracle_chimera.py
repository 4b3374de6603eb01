"""Pins of the Chimera oracle (NEXT row f3, reading F-6; oracle/chimera.py):

* a hand-worked two-stage timeline (tests/golden/chimera_two_stage.txt): M = 2, one micro-batch in
  each direction, T = 10 against DAPPLE's 17 on the same partition, and T = 14 with a sync term;
* M = 1 with weightless layers is DAPPLE with M = 1 (oracle.schedules, the flushed-schedule oracle);
* a record with a replicated stage is not a Chimera partition (UINT64_MAX);
* the executed timeline is a valid schedule: every op starts after its input arrived and after the
  previous op of its worker, each worker runs one op at a time, every op runs once;
* T >= each worker's total work, and T <= the serial sum of every op, transfer and sync.
"""
import os

import numpy as np
import pytest

import workloads as W
from oracle import chimera as CH
from oracle import schedules as SC
from oracle.model import U64_MAX, Partition, encode_partition

HERE = os.path.dirname(os.path.abspath(__file__))


def _golden():
    rows = {}
    with open(os.path.join(HERE, "golden", "chimera_two_stage.txt")) as fh:
        for line in fh:
            line = line.strip()
            if line and not line.startswith("#"):
                k, v = line.split("=")
                rows[k.strip()] = int(v)
    return rows


def test_two_stage_golden():
    g = _golden()
    prof = W.Profile("c", [0, 0], [0, 0], [0, 0], [1, 3], [2, 4])
    st = W.State([[1, 3], [1, 3]], [[2, 4], [2, 4]], [[0, 10**6], [10**6, 0]])
    part = Partition(2, [0], [[0], [1]])
    ops, T = CH.chimera_events(prof, st, part, 2)
    assert T == g["T_M2"]
    assert SC.flush_makespan(prof, st, part, SC.DAPPLE, 2) == g["T_dapple_M2"]
    want = {(0, 0, "F", 0): (0, 1), (1, 1, "F", 0): (0, 1), (0, 1, "F", 1): (1, 4), (1, 0, "F", 1): (1, 4),
            (0, 1, "B", 1): (4, 8), (1, 0, "B", 1): (4, 8), (0, 0, "B", 0): (8, 10), (1, 1, "B", 0): (8, 10)}
    assert {(w, p, k, s): (a, b) for (w, p, k, s, _, a, b) in ops} == want
    prof2 = W.Profile("c", [0, 0], [0, 0], [4, 0], [1, 3], [2, 4])
    assert CH.time_ns(prof2, st, part, 2) == g["T_M2_sync"]


@pytest.mark.parametrize("seed", range(5))
def test_single_micro_batch_is_dapple(seed):
    rng = np.random.default_rng(1400 + seed)
    for _ in range(6):
        L = int(rng.integers(1, 10))
        N = int(rng.integers(1, 8))
        S = int(rng.integers(1, min(N, L) + 1))
        prof = W.random_profile(L, rng, f_max=900, bytes_max=10**5)
        prof = W.Profile(prof.name, prof.O, prof.G, [0] * L, prof.f_ref, prof.b_ref)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        cuts = sorted(int(x) for x in rng.choice(L - 1, S - 1, replace=False)) if S > 1 else []
        ws = [int(x) for x in rng.permutation(N)[:S]]
        part = Partition(S, cuts, [[w] for w in ws])
        assert CH.time_ns(prof, st, part, 1) == SC.flush_makespan(prof, st, part, SC.DAPPLE, 1)


def test_replicated_stage_is_not_chimera():
    prof = W.toy()
    st = W.toy_state()
    part = Partition(2, [3], [[0, 1], [2]])
    assert CH.time_ns(prof, st, part, 4) == U64_MAX
    assert CH.score_record(prof, st, encode_partition(part), 4) == U64_MAX


@pytest.mark.parametrize("seed", range(5))
def test_timeline_valid_and_bounds(seed):
    rng = np.random.default_rng(1500 + seed)
    for _ in range(5):
        L = int(rng.integers(2, 10))
        N = int(rng.integers(2, 9))
        S = int(rng.integers(1, min(N, L, 8) + 1))
        M = int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=900, bytes_max=10**5)
        st = W.random_state_small(prof, N, rng, tau_max=3000)
        cuts = sorted(int(x) for x in rng.choice(L - 1, S - 1, replace=False)) if S > 1 else []
        ws = [int(x) for x in rng.permutation(N)[:S]]
        part = Partition(S, cuts, [[w] for w in ws])
        ops, T = CH.chimera_events(prof, st, part, M)
        assert len(ops) == 2 * S * M
        busy = {}
        prev_end = {}
        for (w, pipe, kind, s, k, a, b) in ops:
            assert a >= prev_end.get(w, 0)       # one op at a time, in execution order
            prev_end[w] = b
            busy[w] = busy.get(w, 0) + (b - a)
        assert T >= max(busy.values())
        assert T >= max(b for (*_, b) in ops)
        serial = sum(b - a for (*_, a, b) in ops)
        stages = part.stage_layers(L)
        comm = sum(CH.xfer(prof.O[stages[s][1]], max(max(r) for r in st.tau)) +
                   CH.xfer(prof.G[stages[s][1] + 1], max(max(r) for r in st.tau)) for s in range(S - 1)) * M
        sync = sum(SC.ps_duration(prof.P, a, e, sorted({ws[s], ws[S - 1 - s]}), st.tau) +
                   CH.allreduce_duration(prof.P, a, e, sorted({ws[s], ws[S - 1 - s]}), st.tau)
                   for s, (a, e) in enumerate(stages))
        assert T <= serial + comm + sync
