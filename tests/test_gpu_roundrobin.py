"""GPU parity of NEXT row f4's round-robin replicas (autopipe_set_schedule(AUTOPIPE_SCHED_PIPEDREAM_RR);
reading F-5; rr.cuh) against oracle/roundrobin.py, element by element, bit-exact: random records
(replicas, random placement, invalid ones), both sync schemes, the C5 ResNet-50 state, all-r = 1
records (= the PipeDream model), small-space searches (= the oracle's minimum over the enumeration)
and the refused calls."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import roundrobin as RR
from oracle.enumerate import candidates, count
from oracle.model import encode_partition
from tests._oracle_pool import rr_many, score_many

pytestmark = pytest.mark.gpu
SCHED_RR = 4


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


DEFER_MODES = {"default": {}, "defer_all": {"rr_defer_all": True}, "no_defer": {"rr_no_defer": True}}


@pytest.mark.parametrize("mode", list(DEFER_MODES))
@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("sync", [0, 1])
def test_random_records(eng, seed, sync, mode):
    """Every record three ways: the default (simulation, deferral of the slow ones to the warp-per-
    record drain kernel), defer_all (a one-round budget: nearly every record is finished by the
    drain's Bellman-Ford inside the bracket of its first block) and no_defer (in the thread)."""
    rng = np.random.default_rng(1100 + seed)
    eng.set_search_options(**DEFER_MODES[mode])
    for _ in range(3):
        L = int(rng.integers(2, 14))
        N = int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([300, 10**6])), bytes_max=int(rng.choice([10**3, 10**7])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([200, 10**5])))
        eng.load(prof, st)
        eng.set_schedule(SCHED_RR, sync)
        recs = [bytes(r) for r in W.sample_records(L, N, 300, int(rng.integers(1 << 30)))]
        recs += [bytes([3, 5, 1] + [0xFF] * 13)]                      # an invalid record (cuts)
        assert gpu_eval(eng, recs) == rr_many(prof, st, recs, sync)
    eng.set_schedule()
    eng.set_search_options()


def test_r1_records_equal_pipedream(eng):
    rng = np.random.default_rng(1200)
    prof = W.random_profile(12, rng, f_max=10**6, bytes_max=10**7)
    st = W.random_state_small(prof, 8, rng, tau_max=10**5)
    eng.load(prof, st)
    recs = []
    for _ in range(400):
        S = int(rng.integers(1, 9))
        cuts = sorted(int(x) for x in rng.choice(11, S - 1, replace=False))
        ws = [int(x) for x in rng.permutation(8)[:S]]
        sow = [W.IDLE] * 8
        for s, w in enumerate(ws):
            sow[w] = s
        recs.append(W.encode(S, cuts, sow))
    eng.set_schedule(SCHED_RR)
    got = gpu_eval(eng, recs)
    eng.set_schedule()
    assert got == gpu_eval(eng, recs) == score_many(prof, st, recs)


@pytest.mark.parametrize("mode", list(DEFER_MODES))
def test_resnet50_rollout_state(eng, mode):
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    eng.load(prof, st)
    eng.set_schedule(SCHED_RR)
    eng.set_search_options(**DEFER_MODES[mode])
    recs = [bytes(r) for r in W.sample_records(prof.L, st.N, 1500, 31)]
    assert gpu_eval(eng, recs) == rr_many(prof, st, recs)
    eng.set_schedule()
    eng.set_search_options()


@pytest.mark.parametrize("mode", list(DEFER_MODES))
@pytest.mark.parametrize("seed", range(4))
def test_small_space_search(eng, seed, mode):
    rng = np.random.default_rng(1300 + seed)
    L = int(rng.integers(3, 8))
    N = int(rng.integers(2, 6))
    prof = W.random_profile(L, rng, f_max=2000, bytes_max=10**5)
    st = W.random_state_small(prof, N, rng, tau_max=3000)
    eng.load(prof, st)
    smax = min(N, L, 4)
    recs = [encode_partition(p) for p in candidates(L, N, 1, smax, 0)]
    ts = rr_many(prof, st, recs)
    m = min(ts)
    eng.set_schedule(SCHED_RR)
    for split in (False, True):
        eng.set_search_options(split, **DEFER_MODES[mode])
        r = eng.search_optimum(1, smax)
        assert (r.time_ns, r.index, r.evaluated) == (m, ts.index(m), count(L, N, 1, smax))
    eng.set_search_options(False)
    eng.set_schedule()


def test_refused_calls(eng):
    from paper_conf_icpp_hulww24_b200 import AutopipeError
    from paper_conf_icpp_hulww24_b200._lib import AUTOPIPE_E_INVAL
    prof = W.resnet50()
    st = W.testbed_state(prof, seed=10)          # 10 workers
    eng.load(prof, st)
    eng.set_schedule(SCHED_RR)
    recs = W.sample_records(prof.L, 10, 8, 3, s_max=10, wide=True)
    with pytest.raises(AutopipeError) as ex:
        eng.eval_partitions(torch.from_numpy(recs))
    assert ex.value.code == AUTOPIPE_E_INVAL
    with pytest.raises(AutopipeError):
        eng.set_schedule(SCHED_RR, 0, 2)          # M must be 1
    eng.set_schedule()
