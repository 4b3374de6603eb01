"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle, element by element.

Integer times: the bar is bit-exact equality. Inputs are seeded and synthetic (workloads/).
"""
from math import comb

import numpy as np
import pytest
import torch

import workloads as W
from oracle.enumerate import USE_ALL_WORKERS, count, decode, index_of
from oracle.model import encode_partition, parse_record
from oracle.param_dp import optimum
from oracle.search import brute_force
from tests._oracle_pool import rollout_many, score_many

pytestmark = pytest.mark.gpu

U64_MAX = (1 << 64) - 1


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.close()


@pytest.fixture(params=[False, True], ids=["dense", "split"])
def split(request, eng):
    """Both kernel selections of the search (autopipe_set_search_options): the dense launch for
    small ranges (default) and the per-S split (r = 1 sweep + threshold walk) forced."""
    eng.set_search_options(request.param)
    yield request.param
    eng.set_search_options(False)


def gpu_eval(eng, recs):
    from paper_conf_icpp_hulww24_b200 import as_u64
    if isinstance(recs, np.ndarray):
        arr = np.ascontiguousarray(recs, dtype=np.uint8).reshape(-1, 16)
    else:
        arr = np.frombuffer(b"".join(bytes(r) for r in recs), dtype=np.uint8).reshape(-1, 16).copy()
    t = torch.from_numpy(arr)
    out = as_u64(eng.eval_partitions(t))
    torch.cuda.synchronize()
    return [int(x) for x in out]


def records_of_indices(L, N, smin, smax, flags, idxs):
    return [encode_partition(decode(L, N, smin, smax, flags, int(i))) for i in idxs]


# ------------------------------------------------------------------------------------------------
# toy config: every candidate, the search, the index decode
# ------------------------------------------------------------------------------------------------

def test_toy_every_candidate(eng):
    prof, st = W.toy(), W.toy_state()
    eng.load(prof, st)
    n = count(8, 4, 1, 4)
    recs = records_of_indices(8, 4, 1, 4, 0, range(n))
    assert gpu_eval(eng, recs) == score_many(prof, st, recs)


@pytest.mark.parametrize("flags", [0, USE_ALL_WORKERS])
def test_toy_search(eng, flags, split):
    prof, st = W.toy(), W.toy_state()
    eng.load(prof, st)
    T, idx, part, n = brute_force(prof, st, 1, 4, flags)
    r = eng.search_optimum(1, 4, flags)
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, n)
    assert r.partition == encode_partition(part)
    assert eng.count_candidates(1, 4, flags) == n


def test_decode_index_matches_oracle(eng):
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    rng = np.random.default_rng(4)
    for flags in (0, USE_ALL_WORKERS):
        total = count(21, 8, 1, 8, flags)
        for i in list(rng.integers(0, total, size=200)) + [0, total - 1]:
            assert eng.decode_index(1, 8, flags, int(i)) == encode_partition(decode(21, 8, 1, 8, flags, int(i)))


# ------------------------------------------------------------------------------------------------
# random small instances: explicit records (replicas, random placement, invalid records)
# ------------------------------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(6))
def test_random_records(eng, seed):
    rng = np.random.default_rng(100 + seed)
    for it in range(8):
        L = int(rng.integers(1, 40))
        N = int(rng.integers(1, 9))
        scale = int(rng.choice([10, 10**6, 10**9]))
        prof = W.random_profile(L, rng, f_max=scale, bytes_max=int(rng.choice([10, 10**6, 10**9])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([10, 10**4, 10**6])))
        st.f = [[int(x) * scale // 1000 for x in row] for row in st.f]
        st.b = [[int(x) * scale // 1000 for x in row] for row in st.b]
        eng.load(prof, st)
        recs = W.sample_records(L, N, 300, seed * 100 + it)
        recs = W.corrupt_records(recs, L, N, seed * 100 + it)
        recs = [bytes(r) for r in recs]
        assert gpu_eval(eng, recs) == score_many(prof, st, recs)


def test_invalid_records(eng):
    prof, st = W.toy(), W.toy_state()
    eng.load(prof, st)
    bad = [W.encode(0, [], [0, 0, 0, 0]), W.encode(5, [1, 2, 3, 4], [0, 1, 2, 3]),
           W.encode(2, [7], [0, 1, 1, 1]), W.encode(3, [4, 4], [0, 1, 2, 2]),
           W.encode(2, [3], [0, 0, 0, W.IDLE]), W.encode(2, [3], [0, 1, 1, 1, 0]),
           W.encode(2, [3], [0, 2, 1, 1]), bytes([1] + [0xFF] * 15)]
    assert gpu_eval(eng, bad) == [U64_MAX] * len(bad)


# ------------------------------------------------------------------------------------------------
# search: brute force on small spaces, shards, both flags
# ------------------------------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(4))
def test_random_search_and_shards(eng, seed, split):
    rng = np.random.default_rng(200 + seed)
    for it in range(5):
        L = int(rng.integers(2, 12))
        N = int(rng.integers(1, 6))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([50, 10**6])), bytes_max=int(rng.choice([100, 10**7])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([100, 10**5])))
        eng.load(prof, st)
        flags = int(rng.integers(0, 2))
        smax = min(N, 8)
        smin = int(rng.integers(1, smax + 1))
        total = count(L, N, smin, smax, flags)
        if total == 0:
            continue
        T, idx, part, n = brute_force(prof, st, smin, smax, flags)
        r = eng.search_optimum(smin, smax, flags)
        assert (r.time_ns, r.index, r.evaluated) == (T, idx, n)
        # a random shard
        b = int(rng.integers(0, total))
        e = int(rng.integers(b, total + 1))
        T2, idx2, _, n2 = brute_force(prof, st, smin, smax, flags, begin=b, end=e)
        r2 = eng.search_optimum(smin, smax, flags, begin=b, end=e)
        if n2 == 0:
            assert r2.empty and r2.evaluated == 0
        else:
            assert (r2.time_ns, r2.index, r2.evaluated) == (T2, idx2, n2)


# ------------------------------------------------------------------------------------------------
# the paper-shaped configs: seeded samples vs the oracle, optima vs the param DP
# ------------------------------------------------------------------------------------------------

def _sample_parity(eng, prof, st, smin, smax, flags, n, seed):
    L, N = prof.L, st.N
    total = count(L, N, smin, smax, flags)
    rng = np.random.default_rng(seed)
    idxs = rng.integers(0, total, size=n)
    recs = records_of_indices(L, N, smin, smax, flags, idxs)
    assert gpu_eval(eng, recs) == score_many(prof, st, recs)


def test_vgg16_sample_and_optimum(eng, split):
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    _sample_parity(eng, prof, st, 1, 8, 0, 10_000, 12345)
    r = eng.search_optimum(1, 8)
    T, idx, part = optimum(prof, st, 1, 8)
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, 1_184_040)
    assert r.partition == encode_partition(part)
    assert score_many(prof, st, [r.partition])[0] == T


def test_vgg16_random_placement_records(eng):
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    recs = [bytes(x) for x in W.sample_records(prof.L, st.N, 5000, 12345)]
    assert gpu_eval(eng, recs) == score_many(prof, st, recs)


@pytest.mark.parametrize("name", ["gnmt16", "bert24"])
def test_trace_states(eng, name, split):
    """C3: the fluctuation trace re-scored per state switch; each optimum equals the param DP."""
    prof = W.profile(name)
    for st in W.trace_c3(prof):
        eng.load(prof, st)
        smax = min(8, st.N)
        r = eng.search_optimum(1, smax)
        T, idx, part = optimum(prof, st, 1, smax)
        assert (r.time_ns, r.index) == (T, idx), st.label
        assert r.evaluated == count(prof.L, st.N, 1, smax)
    _sample_parity(eng, prof, st, 1, smax, 0, 2000, 12345)


@pytest.mark.parametrize("kind", ["a-nvlink", "b"])
def test_gpt96_full_search(eng, kind):
    """C4: the exhaustive 96-layer, 8-stage space (C(95,7) = 1.1e10 candidates)."""
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load(prof, st)
    assert eng.int_path == (32 if kind.startswith("a") else 64)
    r = eng.search_optimum(8, 8)
    T, idx, part = optimum(prof, st, 8, 8)
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, comb(95, 7))
    assert r.partition == encode_partition(part)
    _sample_parity(eng, prof, st, 8, 8, 0, 2000, 12345)


def test_gpt96_shards_match(eng):
    """8 shards of the 1.1e10 space, min-loc reduced on the host, equal the single search."""
    prof, st = W.gpt96(), W.gpt_state("a-100g")
    eng.load(prof, st)
    total = comb(95, 7)
    full = eng.search_optimum(8, 8)
    parts = [eng.search_optimum(8, 8, begin=r * total // 8, end=(r + 1) * total // 8) for r in range(8)]
    best = min(parts, key=lambda p: (p.time_ns, p.index))
    assert (best.time_ns, best.index) == (full.time_ns, full.index)
    assert sum(p.evaluated for p in parts) == total


# ------------------------------------------------------------------------------------------------
# rollouts (C5) and error paths
# ------------------------------------------------------------------------------------------------

def test_rollout_rewards(eng):
    from paper_conf_icpp_hulww24_b200 import as_u64
    prof = W.resnet50()
    for step in range(3):
        st = W.rollout_state(prof, step)
        eng.load(prof, st)
        recs = W.sample_records(prof.L, st.N, 3000, 1000 + step)
        cur = bytes(recs[0])
        t, sw = eng.rollout_rewards(torch.from_numpy(recs), cur)
        torch.cuda.synchronize()
        ot, osw = rollout_many(prof, st, [bytes(r) for r in recs], cur)
        assert [int(x) for x in as_u64(t)] == ot
        assert [int(x) for x in as_u64(sw)] == osw
        t2, sw2 = eng.rollout_rewards(torch.from_numpy(recs), None)
        assert sw2 is None and [int(x) for x in as_u64(t2)] == ot


def test_error_paths():
    from paper_conf_icpp_hulww24_b200 import AutopipeError, Engine
    from paper_conf_icpp_hulww24_b200._lib import (AUTOPIPE_E_INVAL, AUTOPIPE_E_OVERFLOW,
                                                   AUTOPIPE_E_STATE)
    e = Engine(0)
    with pytest.raises(AutopipeError) as ex:
        e.search_optimum(1, 1)
    assert ex.value.code == AUTOPIPE_E_STATE
    prof, st = W.toy(), W.toy_state()
    e.load_profile(prof.O, prof.G, prof.P)
    with pytest.raises(AutopipeError) as ex:
        e.eval_partitions(torch.zeros((1, 16), dtype=torch.uint8))
    assert ex.value.code == AUTOPIPE_E_STATE
    e.set_state(st.f, st.b, st.tau)
    with pytest.raises(AutopipeError) as ex:
        e.search_optimum(0, 2)
    assert ex.value.code == AUTOPIPE_E_INVAL
    with pytest.raises(AutopipeError) as ex:
        e.search_optimum(1, 5)
    assert ex.value.code == AUTOPIPE_E_INVAL
    with pytest.raises(AutopipeError) as ex:
        e.rollout_rewards(torch.zeros((1, 16), dtype=torch.uint8), W.encode(0, [], [0] * 4))
    assert ex.value.code == AUTOPIPE_E_INVAL
    # bytes * tau >= 2^64
    with pytest.raises(AutopipeError) as ex:
        e.set_state(st.f, st.b, [[0 if u == v else (1 << 50) for v in range(4)] for u in range(4)])
    assert ex.value.code == AUTOPIPE_E_OVERFLOW
    # times reaching 2^59 ns
    with pytest.raises(AutopipeError) as ex:
        e.set_state([[1 << 58] * 8] * 4, st.b, st.tau)
    assert ex.value.code == AUTOPIPE_E_OVERFLOW
    with pytest.raises(AutopipeError) as ex:
        e.load_profile([1 << 57], [0], [0])
    assert ex.value.code == AUTOPIPE_E_OVERFLOW
    e.close()


def test_near_overflow_values_exact(eng):
    """Values close to the 2^59 bound still score bit-exactly (u64 path, ceil divisions by r <= 8)."""
    rng = np.random.default_rng(9)
    L, N = 6, 8
    big = (1 << 59) // (2 * L * 4)
    prof = W.Profile("big", [int(x) for x in rng.integers(0, 1 << 40, L)],
                     [int(x) for x in rng.integers(0, 1 << 40, L)],
                     [int(x) for x in rng.integers(0, 1 << 40, L)], [1] * L, [1] * L)
    st = W.State([[int(x) for x in rng.integers(big // 2, big, L)] for _ in range(N)],
                 [[int(x) for x in rng.integers(big // 2, big, L)] for _ in range(N)],
                 [[0 if u == v else int(rng.integers(1, 4000)) for v in range(N)] for u in range(N)])
    eng.load(prof, st)
    assert eng.int_path == 64
    recs = [bytes(r) for r in W.sample_records(L, N, 2000, 77)]
    assert gpu_eval(eng, recs) == score_many(prof, st, recs)


# ------------------------------------------------------------------------------------------------
# the hot r = 1 kernel (S >= 5): shards with partial rows and heavy ties, against the oracle's event
# simulation of every candidate and the parametric DP
# ------------------------------------------------------------------------------------------------

def _all_records(L, N, smin, smax, flags):
    from oracle.enumerate import candidates
    return [encode_partition(p) for p in candidates(L, N, smin, smax, flags)]


@pytest.mark.parametrize("S,L,uniform", [(5, 22, False), (6, 24, True), (7, 20, False), (8, 19, True)])
def test_r1_kernel_shards_and_ties(eng, S, L, uniform, split):
    rng = np.random.default_rng(300 + S)
    if uniform:   # identical layers and workers: huge numbers of exact ties in T
        prof = W.Profile("u", [1000] * L, [1000] * L, [0] * L, [7] * L, [13] * L)
        st = W.State([[7] * L] * S, [[13] * L] * S, [[0 if u == v else 5000 for v in range(S)] for u in range(S)])
    else:
        prof = W.random_profile(L, rng, f_max=10**6, bytes_max=10**7)
        st = W.random_state_small(prof, S, rng, tau_max=10**5)
        st.f = [[x * 1000 for x in row] for row in st.f]
        st.b = [[x * 1000 for x in row] for row in st.b]
    eng.load(prof, st)
    recs = _all_records(L, S, S, S, USE_ALL_WORKERS)       # exactly the r = 1 block
    times = np.array(score_many(prof, st, recs), dtype=object)
    total = len(recs)
    full = eng.search_optimum(S, S, USE_ALL_WORKERS)
    T, idx, _ = optimum(prof, st, S, S, USE_ALL_WORKERS)
    assert (full.time_ns, full.index, full.evaluated) == (T, idx, total)
    for _ in range(12):
        b = int(rng.integers(0, total))
        e = int(rng.integers(b + 1, total + 1))
        sub = times[b:e]
        m = min(sub)
        want = (m, b + list(sub).index(m), e - b)
        r = eng.search_optimum(S, S, USE_ALL_WORKERS, begin=b, end=e)
        assert (r.time_ns, r.index, r.evaluated) == want, (b, e)


@pytest.mark.parametrize("kind", ["a-nvlink", "b"])
def test_gpt96_shard_boundaries_vs_oracle(eng, kind, split):
    """Full size, in the launch configuration bench.py times: the 96-layer, 8-stage space split into
    the 8 cost-balanced shards of the multi-GPU split. Around every inner shard boundary a window of
    candidates straddling it is searched on the GPU as two pieces (the end of the left shard, the
    start of the right one: partial rows on both sides) and each piece is compared with the oracle's
    brute force over the same indices; the shard holding the optimum returns the parametric DP's
    optimum."""
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load(prof, st)
    total = comb(95, 7)
    b = balanced_bounds(96, 8, 8, 8, 0, 8)
    half = 1500
    for i in range(1, 8):
        lo, mid, hi = b[i] - half, b[i], b[i] + half
        recs = records_of_indices(96, 8, 8, 8, 0, range(lo, hi))
        ts = score_many(prof, st, recs)
        for a, e in ((lo, mid), (mid, hi)):
            sub = ts[a - lo:e - lo]
            m = min(sub)
            want = (m, a + sub.index(m), e - a)
            r = eng.search_optimum(8, 8, begin=a, end=e)
            assert (r.time_ns, r.index, r.evaluated) == want, (kind, i, a, e)
    T, idx = optimum(prof, st, 8, 8)[:2]
    k = next(i for i in range(8) if b[i] <= idx < b[i + 1])
    r = eng.search_optimum(8, 8, begin=b[k], end=b[k + 1])
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, b[k + 1] - b[k])
    assert sum(eng.search_optimum(8, 8, begin=b[j], end=b[j + 1]).evaluated for j in range(8)) == total


def test_set_state_device_matches_host(eng):
    prof, st = W.gpt96(), W.gpt_state("b")
    eng.load(prof, st)
    host = eng.search_optimum(8, 8, begin=10**9, end=2 * 10**9)
    dev = torch.device("cuda", 0)
    as_t = lambda a: torch.tensor(np.asarray(a, dtype=np.uint64).view(np.int64), device=dev)
    eng.set_state_device(as_t(st.f), as_t(st.b), as_t(st.tau))
    assert eng.int_path == 64
    devr = eng.search_optimum(8, 8, begin=10**9, end=2 * 10**9)
    assert (devr.time_ns, devr.index, devr.evaluated) == (host.time_ns, host.index, host.evaluated)
    recs = W.sample_records(prof.L, st.N, 500, 5)
    assert gpu_eval(eng, recs) == score_many(prof, st, [bytes(r) for r in recs])


def test_set_state_device_overflow(eng):
    from paper_conf_icpp_hulww24_b200 import AutopipeError
    from paper_conf_icpp_hulww24_b200._lib import AUTOPIPE_E_OVERFLOW
    prof, st = W.toy(), W.toy_state()
    eng.load(prof, st)
    dev = torch.device("cuda", 0)
    big = torch.full((4, 8), 1 << 58, dtype=torch.int64, device=dev)
    tau = torch.tensor(np.asarray(st.tau, dtype=np.int64), device=dev)
    eng.set_state_device(big, big, tau)
    assert gpu_eval(eng, [W.encode(1, [], [0, W.IDLE, W.IDLE, W.IDLE])]) == [U64_MAX]
    with pytest.raises(AutopipeError) as ex:
        eng.search_optimum(1, 2)
    assert ex.value.code == AUTOPIPE_E_OVERFLOW


# ------------------------------------------------------------------------------------------------
# NEXT row f1: the two-worker neighbourhood against the oracle's definition
# ------------------------------------------------------------------------------------------------

@pytest.mark.parametrize("seed", range(4))
def test_neighbourhood_matches_oracle(eng, seed):
    from oracle.neighbourhood import all_partitions, best_neighbour, neighbourhood
    rng = np.random.default_rng(500 + seed)
    for it in range(4):
        L = int(rng.integers(2, 8))
        N = int(rng.integers(1, 5))
        prof = W.random_profile(L, rng, f_max=1000, bytes_max=10**6)
        st = W.random_state_small(prof, N, rng, tau_max=10**4)
        eng.load(prof, st)
        parts = list(all_partitions(L, N))
        for k in rng.choice(len(parts), size=min(4, len(parts)), replace=False):
            cur = encode_partition(parts[int(k)])
            got = eng.neighbourhood(cur).cpu().numpy()
            got = sorted(bytes(r) for r in got)
            assert got == neighbourhood(L, N, parts[int(k)])
            T, rec, n = best_neighbour(prof, st, cur)
            r = eng.best_neighbour(cur)
            assert (r.time_ns, r.partition, r.evaluated) == (T, rec, n)


def test_neighbourhood_gpt96_and_local_search(eng):
    """On the 96-layer space: every listed neighbour is a valid partition at distance 1 or 2 from
    the current one by the oracle's definition (per-worker layer sets, reading F-1), none twice; the
    listing contains every single-boundary move (each inner cut shifted to every position between
    its neighbours: distance 2, enumerated independently here); a sample is scored by the oracle;
    the best equals the minimum over the listed neighbours, and the paper's gradual migration from
    the even split strictly descends and never beats the exhaustive optimum."""
    from oracle.neighbourhood import layer_sets
    prof, st = W.gpt96(), W.gpt_state("b")
    eng.load(prof, st)
    cuts = [11, 23, 35, 47, 59, 71, 83]
    even = W.contiguous_record(96, cuts, [1] * 8)
    nb = eng.neighbourhood(even)
    t = [int(x) for x in as_u64_list(eng.eval_partitions(nb))]
    recs = [bytes(r) for r in nb.cpu().numpy()]
    assert len(set(recs)) == len(recs)
    base = layer_sets(parse_record(even, 96, 8), 96, 8)
    for rec in recs:
        q = parse_record(rec, 96, 8)
        assert q is not None
        d = sum(1 for x, y in zip(layer_sets(q, 96, 8), base) if x != y)
        assert 1 <= d <= 2
    have = set(recs)
    for j in range(7):
        lo = cuts[j - 1] + 1 if j > 0 else 0
        hi = cuts[j + 1] - 1 if j < 6 else 94
        for c in range(lo, hi + 1):
            if c != cuts[j]:
                moved = cuts[:j] + [c] + cuts[j + 1:]
                assert W.contiguous_record(96, moved, [1] * 8) in have, (j, c)
    rng = np.random.default_rng(41)
    pick = sorted(int(x) for x in rng.choice(len(recs), size=min(200, len(recs)), replace=False))
    assert score_many(prof, st, [recs[i] for i in pick]) == [t[i] for i in pick]
    best = min(zip(t, recs))
    r = eng.best_neighbour(even)
    assert (r.time_ns, r.partition, r.evaluated) == (best[0], best[1], len(recs))
    path = eng.local_search(even, max_steps=200)
    assert all(a[0] > b[0] for a, b in zip(path, path[1:]))
    opt = eng.search_optimum(8, 8)
    assert path[-1][0] >= opt.time_ns
    assert score_many(prof, st, [path[-1][1]])[0] == path[-1][0]


def as_u64_list(t):
    from paper_conf_icpp_hulww24_b200 import as_u64
    torch.cuda.synchronize()
    return as_u64(t)


@pytest.mark.parametrize("kind", ["a-nvlink", "b"])
def test_gpt96_threshold_walk_full_space(eng, kind):
    """The threshold walk (k_search_dfs) over the whole 96-layer, 8-stage space in place of the r = 1
    sweep (AUTOPIPE_SEARCH_NO_R1): the same optimum as the parametric DP, every candidate counted."""
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load(prof, st)
    eng.set_search_options(False, True)
    try:
        r = eng.search_optimum(8, 8)
    finally:
        eng.set_search_options(False)
    T, idx, _ = optimum(prof, st, 8, 8)
    assert (r.time_ns, r.index, r.evaluated) == (T, idx, comb(95, 7))


def test_gpt96_r1_records(eng):
    """The records of the bench's full-T roofline (workloads.r1_records: S = 8, one worker per stage,
    uniform cut sets; state C4a, 32-bit path) against the oracle."""
    prof, st = W.gpt96(), W.gpt_state("a-nvlink")
    eng.load(prof, st)
    recs = W.r1_records(prof.L, 8, 600, 5)
    assert all(parse_record(bytes(r), 96, 8) is not None for r in recs)
    assert gpu_eval(eng, recs) == score_many(prof, st, [bytes(r) for r in recs])


@pytest.mark.parametrize("seed", range(3))
def test_local_search_matches_oracle(eng, seed):
    """autopipe_local_search (the paper's gradual migration) equals the same loop
    over the oracle's best_neighbour, step by step, on tiny spaces."""
    from oracle.neighbourhood import all_partitions, best_neighbour
    from oracle.sim import time_ns
    rng = np.random.default_rng(2100 + seed)
    L, N = int(rng.integers(3, 7)), int(rng.integers(2, 5))
    prof = W.random_profile(L, rng, f_max=1000, bytes_max=10**6)
    st = W.random_state_small(prof, N, rng, tau_max=10**4)
    eng.load(prof, st)
    parts = list(all_partitions(L, N))
    start = encode_partition(parts[int(rng.integers(len(parts)))])
    want = [(time_ns(prof, st, parse_record(start, L, N)), start)]
    for _ in range(50):
        T, rec, _ = best_neighbour(prof, st, want[-1][1])
        if T >= want[-1][0]:
            break
        want.append((T, rec))
    assert eng.local_search(start, max_steps=50) == want
