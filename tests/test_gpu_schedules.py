"""GPU parity of NEXT row f3 (schedule variants and PS sync; sched.cuh / eval.cuh through
autopipe_set_schedule + the scoring calls) against oracle/schedules.py, element by element, bit-exact."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import schedules as SC
from oracle.enumerate import USE_ALL_WORKERS, count, decode
from oracle.model import encode_partition
from tests._oracle_pool import sched_many

pytestmark = pytest.mark.gpu

U64_MAX = (1 << 64) - 1

# (schedule, sync, M, recompute) — every schedule with both syncs, several M, GPipe with recompute
MODELS = [(SC.PIPEDREAM, SC.PS, 1, False), (SC.TWO_BW, SC.RING, 1, False), (SC.TWO_BW, SC.RING, 4, False),
          (SC.TWO_BW, SC.PS, 3, False), (SC.GPIPE, SC.RING, 1, False), (SC.GPIPE, SC.RING, 5, False),
          (SC.GPIPE, SC.PS, 4, True), (SC.DAPPLE, SC.RING, 2, False), (SC.DAPPLE, SC.PS, 7, False),
          (SC.DAPPLE, SC.RING, 12, False)]


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.set_schedule()
    e.close()


def gpu_eval(eng, recs, model):
    from paper_conf_icpp_hulww24_b200 import as_u64
    sched, sync, M, rc = model
    eng.set_schedule(sched, sync, M, rc)
    arr = np.ascontiguousarray(np.asarray(recs, dtype=np.uint8).reshape(-1, 16))
    out = as_u64(eng.eval_partitions(torch.from_numpy(arr)))
    torch.cuda.synchronize()
    eng.set_schedule()
    return [int(x) for x in out]


def _recs(L, N, n, seed, p=0.6):
    return W.sample_records(L, N, n, seed, random_placement_p=p)


@pytest.mark.parametrize("model", MODELS, ids=lambda m: "s%d_y%d_M%d_r%d" % (m[0], m[1], m[2], m[3]))
def test_random_small(eng, model):
    """Random profiles and states (independent per-worker f/b, asymmetric links, zeros), records with
    replicas and arbitrary placement, invalid records."""
    rng = np.random.default_rng(1000 + model[0] * 10 + model[2])
    for it in range(4):
        L = int(rng.integers(2, 30))
        N = int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=1000, bytes_max=10**6)
        st = W.random_state_small(prof, N, rng, tau_max=10**4)
        eng.load(prof, st)
        recs = _recs(L, N, 250, 50 + it)
        recs = np.concatenate([recs, W.corrupt_records(recs[:50], L, N, it)])
        assert gpu_eval(eng, recs, model) == sched_many(prof, st, [bytes(r) for r in recs], *model)


@pytest.mark.parametrize("name", ["vgg16", "resnet50", "gnmt16", "bert24"])
def test_paper_profiles(eng, name):
    prof = W.profile(name)
    rng = np.random.default_rng(17)
    st = W.random_state(prof, 8, rng, free_link_p=0.1)
    eng.load(prof, st)
    recs = _recs(prof.L, 8, 150, 41)
    for model in [(SC.PIPEDREAM, SC.PS, 1, False), (SC.TWO_BW, SC.PS, 8, False),
                  (SC.GPIPE, SC.RING, 8, True), (SC.DAPPLE, SC.PS, 16, False)]:
        assert gpu_eval(eng, recs, model) == sched_many(prof, st, [bytes(r) for r in recs], *model)


def test_gpt96_full_size_sample(eng):
    """The 96-layer config at full size: a sample of 8-stage records under each schedule."""
    prof, st = W.gpt96(), W.gpt_state("b")
    eng.load(prof, st)
    recs = _recs(96, 8, 120, 96, p=0.3)
    for model in [(SC.TWO_BW, SC.RING, 16, False), (SC.GPIPE, SC.RING, 32, False),
                  (SC.DAPPLE, SC.RING, 32, False)]:
        assert gpu_eval(eng, recs, model) == sched_many(prof, st, [bytes(r) for r in recs], *model)


def _brute(prof, st, L, N, smin, smax, flags, model):
    n = count(L, N, smin, smax, flags)
    recs = [encode_partition(decode(L, N, smin, smax, flags, i)) for i in range(n)]
    ts = sched_many(prof, st, recs, *model)
    best = min(range(n), key=lambda i: (ts[i], i))
    return ts[best], best, n


@pytest.mark.parametrize("model", [(SC.PIPEDREAM, SC.PS, 1, False), (SC.TWO_BW, SC.RING, 3, False),
                                   (SC.GPIPE, SC.PS, 4, True), (SC.DAPPLE, SC.RING, 6, False)],
                         ids=lambda m: "s%d_y%d_M%d_r%d" % (m[0], m[1], m[2], m[3]))
def test_search_small_spaces(eng, model):
    """Exhaustive search under each schedule = the oracle's minimum over the enumeration (first
    minimum wins), on the toy config and random tiny spaces, with both flags and shards."""
    cases = [(W.toy(), W.toy_state(), 1, 4, 0), (W.toy(), W.toy_state(), 1, 4, USE_ALL_WORKERS)]
    rng = np.random.default_rng(23 + model[0])
    for _ in range(3):
        L, N = int(rng.integers(3, 8)), int(rng.integers(2, 5))
        prof = W.random_profile(L, rng, f_max=400, bytes_max=10**5)
        cases.append((prof, W.random_state_small(prof, N, rng, tau_max=4000), 1, min(N, L), 0))
    for prof, st, smin, smax, flags in cases:
        eng.load(prof, st)
        T, idx, n = _brute(prof, st, prof.L, st.N, smin, smax, flags, model)
        eng.set_schedule(*model)
        r = eng.search_optimum(smin, smax, flags)
        mid = n // 3
        a, b = eng.search_optimum(smin, smax, flags, 0, mid), eng.search_optimum(smin, smax, flags, mid)
        eng.set_schedule()
        assert (r.time_ns, r.index, r.evaluated) == (T, idx, n)
        assert min((a.time_ns, a.index), (b.time_ns, b.index)) == (T, idx)
        assert r.partition == encode_partition(decode(prof.L, st.N, smin, smax, flags, idx))


def test_search_gpt96_eight_stage_slice(eng):
    """S = 5..8 spaces route to the fast r = 1 kernel under PipeDream only; under 2BW the generic
    kernel scores the same block: a slice of the GPT-96 space checked against the oracle's values."""
    prof, st = W.gpt96(), W.gpt_state("a-nvlink")
    eng.load(prof, st)
    n0, n1 = 5_000_000_000, 5_000_000_300
    model = (SC.TWO_BW, SC.RING, 2, False)
    eng.set_schedule(*model)
    r = eng.search_optimum(8, 8, 0, n0, n1)
    eng.set_schedule()
    recs = [encode_partition(decode(96, 8, 8, 8, 0, i)) for i in range(n0, n1)]
    ts = sched_many(prof, st, recs, *model)
    best = min(range(len(ts)), key=lambda i: (ts[i], i))
    assert (r.time_ns, r.index, r.evaluated) == (ts[best], n0 + best, n1 - n0)


def test_rollout_and_neighbourhood_follow_the_schedule(eng):
    from paper_conf_icpp_hulww24_b200 import as_u64
    prof = W.resnet50()
    st = W.rollout_state(prof, 3)
    eng.load(prof, st)
    recs = torch.from_numpy(_recs(prof.L, st.N, 300, 5))
    cur = bytes(recs[0].numpy())
    model = (SC.DAPPLE, SC.PS, 4, False)
    t_eval = gpu_eval(eng, recs.numpy(), model)
    eng.set_schedule(*model)
    t, sw = eng.rollout_rewards(recs, cur)
    t_nosw, _ = eng.rollout_rewards(recs)
    best = eng.best_neighbour(cur)
    nb = eng.neighbourhood(cur)
    t_nb = [int(x) for x in as_u64(eng.eval_partitions(nb))]
    eng.set_schedule()
    _, sw_pd = eng.rollout_rewards(recs, cur)
    assert [int(x) for x in as_u64(t)] == t_eval == [int(x) for x in as_u64(t_nosw)]
    assert np.array_equal(as_u64(sw), as_u64(sw_pd))   # switch bytes do not depend on the schedule
    recs_nb = nb.cpu().numpy()
    i = min(range(len(t_nb)), key=lambda k: (t_nb[k], bytes(recs_nb[k])))
    assert (best.time_ns, best.partition) == (t_nb[i], bytes(recs_nb[i]))
    assert t_nb == sched_many(prof, st, [bytes(r) for r in recs_nb], *model)


def test_device_state(eng):
    prof, st = W.gnmt16(), W.trace_c3(W.gnmt16())[4]
    eng.load(prof, st)
    recs = _recs(prof.L, st.N, 300, 9)
    model = (SC.GPIPE, SC.RING, 6, True)
    ref = gpu_eval(eng, recs, model)
    dev = lambda a: torch.tensor(a, dtype=torch.int64, device="cuda")
    eng.set_state_device(dev(st.f), dev(st.b), dev(st.tau))
    assert gpu_eval(eng, recs, model) == ref


def test_errors_and_setting(eng):
    from paper_conf_icpp_hulww24_b200 import AutopipeError
    from paper_conf_icpp_hulww24_b200._lib import AUTOPIPE_E_INVAL, AUTOPIPE_E_OVERFLOW, AUTOPIPE_E_STATE
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    for bad in [(6, 0, 1, False), (4, 0, 2, False), (0, 2, 1, False), (0, 0, 2, False), (1, 0, 0, False),
                (1, 0, 65537, False), (SC.DAPPLE, 0, 4, True), (SC.TWO_BW, 0, 4, True)]:
        with pytest.raises(AutopipeError) as ex:
            eng.set_schedule(*bad)
        assert ex.value.code == AUTOPIPE_E_INVAL
    eng.set_schedule(SC.GPIPE, SC.PS, 9, True)
    assert eng.get_schedule() == (SC.GPIPE, SC.PS, 9, True)
    eng.load(prof, st)                        # the setting belongs to the context
    assert eng.get_schedule() == (SC.GPIPE, SC.PS, 9, True)
    recs = torch.from_numpy(_recs(prof.L, 8, 20, 1))
    with pytest.raises(AutopipeError) as ex:
        eng.switch_rewards(recs, bytes(recs[0].numpy()), 4)
    assert ex.value.code == AUTOPIPE_E_STATE
    # 16 (M + 1) x bound must stay below 2^63
    big = W.State([[1 << 40] * prof.L] * 8, [[1 << 40] * prof.L] * 8, st.tau)
    eng.set_state(big.f, big.b, big.tau)
    eng.set_schedule(SC.DAPPLE, SC.RING, 65536)
    with pytest.raises(AutopipeError) as ex:
        eng.eval_partitions(recs)
    assert ex.value.code == AUTOPIPE_E_OVERFLOW
    with pytest.raises(AutopipeError) as ex:
        eng.search_optimum(1, 2)
    assert ex.value.code == AUTOPIPE_E_OVERFLOW
    eng.set_schedule()
    eng.eval_partitions(recs)                 # PipeDream: fine with the same state
    torch.cuda.synchronize()
