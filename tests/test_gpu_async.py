"""GPU: the asynchronous search (autopipe_search_optimum_async), the device-side path choice for a
state set from device memory, the device min-loc of row e (autopipe_reduce_results) and the per-search
kernel timers. Anchored to the oracle (brute force, parametric DP) and to the synchronous search,
which tests/test_gpu_parity.py checks against the oracle."""
from math import comb

import numpy as np
import pytest
import torch

import workloads as W
from oracle.model import encode_partition
from oracle.param_dp import optimum
from oracle.search import brute_force

pytestmark = pytest.mark.gpu

U64_MAX = (1 << 64) - 1
DEV = torch.device("cuda", 0)


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.close()


def _dev(a):
    return torch.tensor(np.asarray(a, dtype=np.uint64).view(np.int64), device=DEV)


def _async(eng, *args, **kw):
    from paper_conf_icpp_hulww24_b200 import result_from_bytes
    out = eng.search_optimum_async(*args, **kw)
    return result_from_bytes(out)  # host copy (synchronises)


def _tuple(r):
    return (r.time_ns, r.index, r.evaluated, r.partition)


def test_toy_async_matches_brute_force(eng):
    prof, st = W.toy(), W.toy_state()
    eng.load(prof, st)
    T, idx, part, n = brute_force(prof, st, 1, 4)
    assert _tuple(_async(eng, 1, 4)) == (T, idx, n, encode_partition(part))
    # shards of it, each the oracle's shard minimum
    for b, e in ((0, 50), (50, 51), (51, 165)):
        T, idx, part, n = brute_force(prof, st, 1, 4, begin=b, end=e)
        assert _tuple(_async(eng, 1, 4, begin=b, end=e)) == (T, idx, n, encode_partition(part))


@pytest.mark.parametrize("kind", ["a-nvlink", "b"])
def test_gpt96_async_device_state_gated_paths(eng, kind):
    """Device state: the host never reads the path back; both kernels are enqueued and the state
    kernel's choice gates them (C4a picks the 32-bit path, C4b the 64-bit one). Full space = the
    oracle's parametric DP; 8 shards reduced on the device = the same."""
    from paper_conf_icpp_hulww24_b200 import reduce_results, result_from_bytes
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load_profile(prof.O, prof.G, prof.P)
    eng.set_state_device(_dev(st.f), _dev(st.b), _dev(st.tau))
    T, idx = optimum(prof, st, 8, 8)[:2]
    r = _async(eng, 8, 8)
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, comb(95, 7))
    b = balanced_bounds(96, 8, 8, 8, 0, 8)
    eng.set_state_device(_dev(st.f), _dev(st.b), _dev(st.tau))
    outs = [eng.search_optimum_async(8, 8, begin=b[i], end=b[i + 1]) for i in range(8)]
    red = result_from_bytes(reduce_results(torch.stack(outs)))
    assert (red.time_ns, red.index, red.evaluated, red.partition) == _tuple(r)
    assert eng.int_path == (32 if kind == "a-nvlink" else 64)   # now read back: the path that ran


def test_async_host_state_equals_sync_vgg_and_bert(eng):
    """Generic kernel (replicated compositions), host state: async = sync on whole spaces and shards."""
    for prof, st in ((W.vgg16(), W.vgg_state()), (W.bert24(), W.trace_c3(W.bert24())[2])):
        smax = min(8, len(st.f))
        eng.load(prof, st)
        n = eng.count_candidates(1, smax)
        for b, e in ((0, n), (n // 3, 2 * n // 3 + 1)):
            assert _tuple(_async(eng, 1, smax, begin=b, end=e)) == _tuple(eng.search_optimum(1, smax, begin=b, end=e))


def test_async_device_state_generic_kernel(eng):
    """Device state through the generic kernel (S < 5 and replicated compositions): gated P32 / P64."""
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    want = eng.search_optimum(1, 8)
    eng.set_state_device(_dev(st.f), _dev(st.b), _dev(st.tau))
    assert _tuple(_async(eng, 1, 8)) == _tuple(want)


def test_async_device_state_overflow_and_empty_shard(eng):
    from paper_conf_icpp_hulww24_b200 import AutopipeError
    from paper_conf_icpp_hulww24_b200._lib import AUTOPIPE_E_OVERFLOW
    prof, st = W.toy(), W.toy_state()
    eng.load(prof, st)
    r = _async(eng, 1, 4, begin=7, end=7)
    assert _tuple(r) == (U64_MAX, U64_MAX, 0, bytes([0xFF] * 16))
    big = torch.full((4, 8), 1 << 58, dtype=torch.int64, device=DEV)
    eng.set_state_device(big, big, _dev(st.tau))
    r = _async(eng, 1, 4)
    assert (r.time_ns, r.index, r.evaluated) == (U64_MAX, U64_MAX, 0)
    with pytest.raises(AutopipeError) as ex:
        eng.search_optimum(1, 4)
    assert ex.value.code == AUTOPIPE_E_OVERFLOW


def test_async_searches_back_to_back_then_times(eng):
    """Many asynchronous searches enqueued without waiting (the schedule staging is reused safely),
    then their kernel times read in one call."""
    from paper_conf_icpp_hulww24_b200 import result_from_bytes
    prof, st = W.gpt96(), W.gpt_state("a-nvlink")
    eng.load(prof, st)
    total = comb(95, 7)
    want = [eng.search_optimum(8, 8, begin=k * total // 12, end=(k + 1) * total // 12) for k in range(12)]
    eng.set_timing(True)
    eng.search_times()
    outs = [eng.search_optimum_async(8, 8, begin=k * total // 12, end=(k + 1) * total // 12) for k in range(12)]
    ts = eng.search_times()
    eng.set_timing(False)
    assert len(ts) == 12 and all(t > 0 for t in ts)
    assert [_tuple(result_from_bytes(o)) for o in outs] == [_tuple(w) for w in want]


def test_reduce_results_definition():
    """autopipe_reduce_results = lexicographic (T, index) minimum, evaluated summed, the first minimal
    entry's record; empties (UINT64_MAX, UINT64_MAX) never win over a real result."""
    from paper_conf_icpp_hulww24_b200 import reduce_results, result_from_bytes
    rng = np.random.default_rng(3)
    for n, width in ((1, 40), (2, 40), (7, 40), (33, 40), (100, 56), (5, 56)):
        rows = []
        for i in range(n):
            if rng.random() < 0.2:
                t = idx = U64_MAX
                cnt = 0
            else:
                t, idx, cnt = int(rng.integers(5, 9)), int(rng.integers(0, 4)), int(rng.integers(0, 1000))
            rec = bytes(rng.integers(0, 256, size=width - 24, dtype=np.uint8))
            rows.append(t.to_bytes(8, "little") + idx.to_bytes(8, "little") + cnt.to_bytes(8, "little") + rec)
        g = torch.tensor(np.frombuffer(b"".join(rows), dtype=np.uint8).reshape(n, width), device=DEV)
        got = result_from_bytes(reduce_results(g))
        key = [(int.from_bytes(r[:8], "little"), int.from_bytes(r[8:16], "little")) for r in rows]
        best = min(range(n), key=lambda i: (key[i], i))
        assert (got.time_ns, got.index) == key[best]
        assert got.evaluated == sum(int.from_bytes(r[16:24], "little") for r in rows)
        assert got.partition == rows[best][24:]


def test_async_wide_testbed(eng):
    """Row f4 through the asynchronous call: the 10-worker testbed VGG-16 space."""
    prof = W.vgg16()
    st = W.testbed_state(prof, seed=10)
    eng.load(prof, st)
    want = eng.search_optimum(1, 10)
    got = _async(eng, 1, 10)
    assert _tuple(got) == _tuple(want) and len(got.partition) == 32


def test_wide_sharded_search_reduced(eng):
    """Row e on a wide space (row f4): cost-balanced shards of the 10-worker testbed space, each
    searched asynchronously, reduced on the device = the single search."""
    from paper_conf_icpp_hulww24_b200 import reduce_results, result_from_bytes
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    prof = W.vgg16()
    st = W.testbed_state(prof, seed=10)
    eng.load(prof, st)
    want = eng.search_optimum(1, 10)
    for G in (2, 3, 8):
        b = balanced_bounds(prof.L, 10, 1, 10, 0, G)
        outs = [eng.search_optimum_async(1, 10, begin=b[i], end=b[i + 1]) for i in range(G)]
        got = result_from_bytes(reduce_results(torch.stack(outs)))
        assert _tuple(got) == _tuple(want)


def _bounded_shards(eng, G, bounds, s_min, s_max):
    """Row e with the cross-shard bound, G shards on one GPU: seed every shard, min-reduce the seeds
    (what NCCL all_reduce MIN does across ranks), search every shard under the bound, reduce."""
    from paper_conf_icpp_hulww24_b200 import reduce_results
    seeds = torch.stack([eng.search_seed_async(s_min, s_max, begin=bounds[i], end=bounds[i + 1]).clone()
                         for i in range(G)])
    u = seeds.cpu().numpy().view(np.uint64).ravel()
    theta = torch.tensor(np.array([u.min()], dtype=np.uint64).view(np.int64), device=DEV)
    eng.set_search_bound(theta)
    try:
        outs = [eng.search_optimum_async(s_min, s_max, begin=bounds[i], end=bounds[i + 1]) for i in range(G)]
        red = reduce_results(torch.stack(outs))
    finally:
        eng.set_search_bound(None)
    return int(u.min()), u, outs, red


@pytest.mark.parametrize("kind", ["a-nvlink", "b"])
def test_gpt96_cross_shard_bound(eng, kind):
    """Row e, cross-shard bound: 8 cost-balanced shards of C(95,7), each seeded, the seeds' minimum
    as every shard's starting bound. The reduction = the oracle's parametric DP optimum with every
    candidate counted; each seed is the exact T of a candidate of its shard (>= the optimum); a shard
    whose result is kept has its own exact minimum (= the unbounded search of that shard)."""
    from paper_conf_icpp_hulww24_b200 import result_from_bytes
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load(prof, st)
    T, idx = optimum(prof, st, 8, 8)[:2]
    b = balanced_bounds(96, 8, 8, 8, 0, 8)
    theta, seeds, outs, red = _bounded_shards(eng, 8, b, 8, 8)
    got = result_from_bytes(red)
    assert (got.time_ns, got.index, got.evaluated) == (T, idx, comb(95, 7))
    assert T <= theta < U64_MAX and all(s >= T for s in seeds)
    for i in range(8):
        r = result_from_bytes(outs[i])
        assert r.evaluated == b[i + 1] - b[i]
        if r.time_ns <= theta:
            want = eng.search_optimum(8, 8, begin=b[i], end=b[i + 1])
            assert _tuple(r) == _tuple(want)
        else:
            assert r.index == U64_MAX or r.time_ns > theta
    # the bound cleared: a shard search is unbounded again
    want = eng.search_optimum(8, 8, begin=b[7], end=b[8])
    assert _tuple(_async(eng, 8, 8, begin=b[7], end=b[8])) == _tuple(want)


def test_cross_shard_bound_small_spaces_and_device_state(eng):
    """Spaces whose r = 1 blocks are too small to seed leave the bound at UINT64_MAX (no filtering);
    a device state (gated paths) under a bound gives the same optimum."""
    from paper_conf_icpp_hulww24_b200 import result_from_bytes
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    want = eng.search_optimum(1, 8)
    b = balanced_bounds(prof.L, 8, 1, 8, 0, 3)
    theta, _, _, red = _bounded_shards(eng, 3, b, 1, 8)
    assert theta == U64_MAX
    assert _tuple(result_from_bytes(red)) == _tuple(want)
    prof, st = W.gpt96(), W.gpt_state("b")
    eng.load_profile(prof.O, prof.G, prof.P)
    eng.set_state_device(_dev(st.f), _dev(st.b), _dev(st.tau))
    T, idx = optimum(prof, st, 8, 8)[:2]
    b = balanced_bounds(96, 8, 8, 8, 0, 4)
    _, _, _, red = _bounded_shards(eng, 4, b, 8, 8)
    got = result_from_bytes(red)
    assert (got.time_ns, got.index, got.evaluated) == (T, idx, comb(95, 7))


def test_cross_shard_bound_retired_by_state_change(eng):
    """A bound is keyed to the state and space it was seeded on: a bound from C4a (optimum below
    C4b's) left set while the context moves to C4b must not filter C4b's search, nor a search of
    another stage range; set_search_bound without a seed on the current state is E_STATE."""
    from paper_conf_icpp_hulww24_b200 import AutopipeError
    prof = W.gpt96()
    sa, sb = W.gpt_state("a-nvlink"), W.gpt_state("b")
    eng.load(prof, sa)
    theta = eng.search_seed_async(8, 8).clone()
    eng.set_search_bound(theta)
    try:
        Tb, ib = optimum(prof, sb, 8, 8)[:2]
        assert int(theta.cpu().numpy().view(np.uint64)[0]) < Tb
        eng.set_state(sb.f, sb.b, sb.tau)
        got = _async(eng, 8, 8)
        assert (got.time_ns, got.index, got.evaluated) == (Tb, ib, comb(95, 7))
        # same state, another stage range: unbounded too
        eng.set_state(sa.f, sa.b, sa.tau)
        theta2 = eng.search_seed_async(8, 8).clone()
        eng.set_search_bound(theta2)
        for s in (5, 6, 7):
            eng.set_search_bound(theta2)
            got = _async(eng, s, s)
            eng.set_search_bound(None)
            want = _async(eng, s, s)
            assert _tuple(got) == _tuple(want) and want.index != U64_MAX
        eng.set_search_bound(theta2)
        eng.set_state(sb.f, sb.b, sb.tau)
        with pytest.raises(AutopipeError):
            eng.set_search_bound(theta2)
    finally:
        eng.set_search_bound(None)
