"""GPU parity of NEXT row f3's Chimera model (autopipe_set_schedule(AUTOPIPE_SCHED_CHIMERA, sync, M);
reading F-6; chimera.cuh) against oracle/chimera.py, element by element, bit-exact: one-worker-per-
stage records (and replicated ones, which are not Chimera partitions), M = 1..9, both sync schemes,
the paper-shaped BERT-24 profile, the hand-worked golden, small-space searches and refused calls."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import chimera as CH
from oracle.enumerate import candidates, count
from oracle.model import Partition, encode_partition
from tests._oracle_pool import chimera_many

pytestmark = pytest.mark.gpu
SCHED_CHIMERA = 5


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.set_schedule()
    e.close()


def gpu_eval(eng, recs):
    from paper_conf_icpp_hulww24_b200 import as_u64
    arr = np.frombuffer(b"".join(bytes(r) for r in recs), dtype=np.uint8).reshape(len(recs), 16).copy()
    out = as_u64(eng.eval_partitions(torch.from_numpy(arr)))
    torch.cuda.synchronize()
    return [int(x) for x in out]


def _chimera_records(rng, L, N, n):
    out = []
    for _ in range(n):
        S = int(rng.integers(1, min(N, L, 8) + 1))
        cuts = sorted(int(x) for x in rng.choice(L - 1, S - 1, replace=False)) if S > 1 else []
        ws = [int(x) for x in rng.permutation(N)[:S]]
        out.append(encode_partition(Partition(S, cuts, [[w] for w in ws])))
    return out


def test_golden(eng):
    prof = W.Profile("c", [0, 0], [0, 0], [4, 0], [1, 3], [2, 4])
    st = W.State([[1, 3], [1, 3]], [[2, 4], [2, 4]], [[0, 10**6], [10**6, 0]])
    eng.load(prof, st)
    eng.set_schedule(SCHED_CHIMERA, 0, 2)
    assert gpu_eval(eng, [encode_partition(Partition(2, [0], [[0], [1]]))]) == [14]
    eng.set_schedule()


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("sync", [0, 1])
def test_random_records(eng, seed, sync):
    rng = np.random.default_rng(1600 + seed)
    for M in (1, 2, 3, int(rng.integers(4, 10))):
        L = int(rng.integers(1, 14))
        N = int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([300, 10**6])), bytes_max=int(rng.choice([10**3, 10**7])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([200, 10**5])))
        eng.load(prof, st)
        eng.set_schedule(SCHED_CHIMERA, sync, M)
        recs = _chimera_records(rng, L, N, 200)
        recs += [bytes(r) for r in W.sample_records(L, N, 40, int(rng.integers(1 << 30)))]   # replicas -> MAX
        assert gpu_eval(eng, recs) == chimera_many(prof, st, recs, M, sync)
    eng.set_schedule()


def test_bert24_profile(eng):
    prof = W.bert24()
    st = W.trace_c3(prof)[7]
    eng.load(prof, st)
    rng = np.random.default_rng(1700)
    recs = _chimera_records(rng, prof.L, st.N, 400)
    eng.set_schedule(SCHED_CHIMERA, 0, 8)
    assert gpu_eval(eng, recs) == chimera_many(prof, st, recs, 8)
    eng.set_schedule()


@pytest.mark.parametrize("seed", range(3))
def test_small_space_search(eng, seed):
    rng = np.random.default_rng(1800 + seed)
    L = int(rng.integers(3, 8))
    N = int(rng.integers(2, 6))
    prof = W.random_profile(L, rng, f_max=2000, bytes_max=10**5)
    st = W.random_state_small(prof, N, rng, tau_max=3000)
    eng.load(prof, st)
    smax = min(N, L, 4)
    M = 4
    recs = [encode_partition(p) for p in candidates(L, N, 1, smax, 0)]
    ts = chimera_many(prof, st, recs, M)
    m = min(ts)
    eng.set_schedule(SCHED_CHIMERA, 0, M)
    for split in (False, True):
        eng.set_search_options(split)
        r = eng.search_optimum(1, smax)
        assert (r.time_ns, r.index, r.evaluated) == (m, ts.index(m), count(L, N, 1, smax))
    eng.set_search_options(False)
    eng.set_schedule()


@pytest.mark.parametrize("name", ["bert24", "resnet50"])
def test_wide_testbed(eng, name):
    """The paper runs its Chimera comparison on the 10-GPU testbed:
    32-byte records with up to 10 stages on 10 heterogeneous workers, M = 8."""
    from paper_conf_icpp_hulww24_b200 import as_u64
    prof = W.profile(name)
    st = W.testbed_state(prof, seed=10)
    eng.load(prof, st)
    rng = np.random.default_rng(1900)
    recs = []
    for _ in range(300):
        S = int(rng.integers(1, 11))
        cuts = sorted(int(x) for x in rng.choice(prof.L - 1, S - 1, replace=False)) if S > 1 else []
        ws = [int(x) for x in rng.permutation(10)[:S]]
        recs.append(encode_partition(Partition(S, cuts, [[w] for w in ws]), wide=True))
    recs += [bytes(r) for r in W.sample_records(prof.L, 10, 30, 5, s_max=10, wide=True)]
    arr = np.frombuffer(b"".join(recs), dtype=np.uint8).reshape(len(recs), 32).copy()
    eng.set_schedule(SCHED_CHIMERA, 1, 8)
    got = [int(x) for x in as_u64(eng.eval_partitions(torch.from_numpy(arr)))]
    eng.set_schedule()
    assert got == chimera_many(prof, st, recs, 8, 1)
