"""GPU parity of NEXT row f4 (32-byte wide records: S <= 16 stages, N <= 16 workers, for the paper's
10-GPU testbed) through the _w calls, against the oracle, element by element,
bit-exact."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import schedules as SC
from oracle.enumerate import USE_ALL_WORKERS, count, decode
from oracle.model import encode_partition, parse_record, switch_bytes
from tests._oracle_pool import rollout_many, sched_many, score_many

pytestmark = pytest.mark.gpu

U64_MAX = (1 << 64) - 1


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.set_schedule()
    e.close()


@pytest.fixture(params=[False, True], ids=["dense", "split"])
def split(request, eng):
    """Both kernel selections of the search: the dense launch (default for small ranges) and the
    per-S split (threshold walk) forced."""
    eng.set_search_options(request.param)
    yield request.param
    eng.set_search_options(False)


def gpu_eval(eng, recs):
    from paper_conf_icpp_hulww24_b200 import as_u64
    if isinstance(recs, list):
        recs = np.frombuffer(b"".join(bytes(r) for r in recs), dtype=np.uint8).reshape(len(recs), -1)
    arr = np.ascontiguousarray(np.asarray(recs, dtype=np.uint8))
    out = as_u64(eng.eval_partitions(torch.from_numpy(arr)))
    torch.cuda.synchronize()
    return [int(x) for x in out]


def _wide(L, N, n, seed, p=0.6, s_max=16):
    return W.sample_records(L, N, n, seed, random_placement_p=p, s_max=s_max, wide=True)


@pytest.mark.parametrize("seed", range(6))
def test_random_wide(eng, seed):
    """Random profiles and states with 9-16 workers (and a few with fewer), wide records with up to 16
    stages, replicas, arbitrary placement, invalid records."""
    rng = np.random.default_rng(1600 + seed)
    for it in range(3):
        L = int(rng.integers(2, 40))
        N = int(rng.integers(9, 17)) if it < 2 else int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=1000, bytes_max=10**6)
        st = W.random_state_small(prof, N, rng, tau_max=10**4)
        eng.load(prof, st)
        recs = _wide(L, N, 250, seed * 10 + it)
        recs = np.concatenate([recs, W.corrupt_records(recs[:60], L, N, seed)])
        assert gpu_eval(eng, recs) == score_many(prof, st, [bytes(r) for r in recs])


@pytest.mark.parametrize("name", ["vgg16", "resnet50", "bert24"])
def test_testbed_profiles(eng, name):
    """The paper's 10-GPU testbed size (10/25/40/100 Gb/s NICs, co-located jobs) on its models."""
    prof = W.profile(name)
    st = W.testbed_state(prof, seed=10)
    eng.load(prof, st)
    recs = _wide(prof.L, 10, 300, 41)
    assert gpu_eval(eng, recs) == score_many(prof, st, [bytes(r) for r in recs])


def test_testbed_schedules(eng):
    """Row f3's schedule variants on wide records (10 workers, up to 10 stages)."""
    from paper_conf_icpp_hulww24_b200 import as_u64
    prof = W.resnet50()
    st = W.testbed_state(prof, seed=11)
    eng.load(prof, st)
    recs = _wide(prof.L, 10, 120, 43)
    for model in [(SC.PIPEDREAM, SC.PS, 1, False), (SC.TWO_BW, SC.RING, 4, False),
                  (SC.GPIPE, SC.PS, 6, True), (SC.DAPPLE, SC.RING, 12, False)]:
        eng.set_schedule(*model)
        got = [int(x) for x in as_u64(eng.eval_partitions(torch.from_numpy(recs)))]
        eng.set_schedule()
        assert got == sched_many(prof, st, [bytes(r) for r in recs], *model)


def test_rollout_wide(eng):
    from paper_conf_icpp_hulww24_b200 import as_u64
    prof = W.gnmt16()
    st = W.testbed_state(prof, seed=12, N=12)
    eng.load(prof, st)
    recs = _wide(prof.L, 12, 300, 44)
    cur = bytes(recs[3])
    t, sw = eng.rollout_rewards(torch.from_numpy(recs), cur)
    ot, osw = rollout_many(prof, st, [bytes(r) for r in recs], cur)
    assert [int(x) for x in as_u64(t)] == ot
    assert [int(x) for x in as_u64(sw)] == osw


def _brute(prof, st, L, N, smin, smax, flags):
    n = count(L, N, smin, smax, flags)
    recs = [encode_partition(decode(L, N, smin, smax, flags, i), wide=True) for i in range(n)]
    ts = score_many(prof, st, recs)
    best = min(range(n), key=lambda i: (ts[i], i))
    return ts[best], best, n, recs[best]


@pytest.mark.parametrize("case", ["n10", "s11", "s15", "s16"])
def test_search_wide_small_spaces(eng, case, split):
    """Wide exhaustive search = the oracle's minimum over the enumeration (first minimum wins), for 10
    workers and for spaces whose stages exceed 8, with both flags and a shard split."""
    rng = np.random.default_rng({"n10": 1, "s11": 2, "s15": 3, "s16": 4}[case])
    L, N, smin, smax = {"n10": (6, 10, 1, 6), "s11": (12, 12, 11, 12), "s15": (17, 16, 15, 15),
                        "s16": (16, 16, 16, 16)}[case]
    prof = W.random_profile(L, rng, f_max=400, bytes_max=10**5)
    st = W.random_state_small(prof, N, rng, tau_max=4000)
    eng.load(prof, st)
    for flags in (0, USE_ALL_WORKERS):
        T, idx, n, rec = _brute(prof, st, L, N, smin, smax, flags)
        r = eng.search_optimum(smin, smax, flags, wide=True)
        assert (r.time_ns, r.index, r.evaluated, r.partition) == (T, idx, n, rec)
        mid = n // 3
        a, b = eng.search_optimum(smin, smax, flags, 0, mid, wide=True), eng.search_optimum(smin, smax, flags, mid, wide=True)
        assert min((a.time_ns, a.index), (b.time_ns, b.index)) == (T, idx)
        assert eng.count_candidates(smin, smax, flags) == n
        for i in (0, n // 2, n - 1):
            assert eng.decode_index(smin, smax, flags, i, wide=True) == encode_partition(
                decode(L, N, smin, smax, flags, i), wide=True)


@pytest.mark.parametrize("name,smax", [("vgg16", 8), ("gnmt16", 8)])
def test_wide_search_equals_16_byte_search(eng, name, smax, split):
    """For N <= 8 the wide search scans the same index order with the same kernels (the fast r = 1
    kernel for S >= 5): same optimum, same index, the record in its wide form."""
    prof = W.profile(name)
    st = W.vgg_state() if name == "vgg16" else W.trace_c3(prof)[3]
    eng.load(prof, st)
    a = eng.search_optimum(1, smax)
    b = eng.search_optimum(1, smax, wide=True)
    assert (a.time_ns, a.index, a.evaluated) == (b.time_ns, b.index, b.evaluated)
    pa = parse_record(a.partition, prof.L, st.N)
    assert encode_partition(pa, wide=True) == b.partition


@pytest.mark.parametrize("name", ["vgg16", "resnet50"])
def test_testbed_search_ten_workers(eng, name):
    """The 10-GPU testbed (row f4): exhaustive S <= 10, sum r <= 10 search of VGG-16 (14.3M
    candidates) and ResNet-50 (12.6e9) on 10 heterogeneous workers, pinned to the oracle's parametric
    DP (value and lexicographically-first index), the optimum re-scored by the oracle's event
    simulation, and a seeded sample of the space checked against it."""
    from oracle.param_dp import optimum
    prof = W.profile(name)
    st = W.testbed_state(prof, seed=10)
    eng.load(prof, st)
    n = eng.count_candidates(1, 10)
    r = eng.search_optimum(1, 10)
    T, idx = optimum(prof, st, 1, 10)[:2]
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, n)
    assert len(r.partition) == 32
    assert r.partition == encode_partition(decode(prof.L, 10, 1, 10, 0, idx), wide=True)
    assert score_many(prof, st, [r.partition]) == [r.time_ns]
    rng = np.random.default_rng(5)
    idx = sorted(int(x) for x in rng.choice(n, size=300, replace=False))
    recs = [encode_partition(decode(prof.L, 10, 1, 10, 0, i), wide=True) for i in idx]
    ts = score_many(prof, st, recs)
    assert min(ts) >= r.time_ns
    assert gpu_eval(eng, recs) == ts


def test_16_byte_calls_with_more_than_8_workers(eng):
    from paper_conf_icpp_hulww24_b200 import AutopipeError
    from paper_conf_icpp_hulww24_b200._lib import AUTOPIPE_E_INVAL
    prof = W.resnet50()
    st = W.testbed_state(prof, seed=13)
    eng.load(prof, st)
    # 16-byte records can still be scored (they name workers < 8)
    recs = W.sample_records(prof.L, 8, 200, 45)
    assert gpu_eval(eng, recs) == score_many(prof, st, [bytes(r) for r in recs])
    for call in (lambda: eng.search_optimum(1, 4, wide=False), lambda: eng.decode_index(1, 4, 0, 0, wide=False),
                 lambda: eng.best_neighbour(bytes(recs[0])),
                 lambda: eng.switch_rewards(torch.from_numpy(recs), bytes(recs[0]), 4)):
        with pytest.raises(AutopipeError) as ex:
            call()
        assert ex.value.code == AUTOPIPE_E_INVAL


def test_device_state_wide(eng):
    prof = W.bert24()
    st = W.testbed_state(prof, seed=14, N=16)
    eng.load(prof, st)
    recs = _wide(prof.L, 16, 300, 46)
    ref = gpu_eval(eng, recs)
    dev = lambda a: torch.tensor(a, dtype=torch.int64, device="cuda")
    eng.set_state_device(dev(st.f), dev(st.b), dev(st.tau))
    assert gpu_eval(eng, recs) == ref
    assert ref == score_many(prof, st, [bytes(r) for r in recs])
