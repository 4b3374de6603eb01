"""GPU parity of NEXT row f2 (switching cost as time; k_switch.cu through autopipe_switch_rewards)
against the oracle (oracle/switching.py), element by element, bit-exact."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle.model import encode_partition, parse_record
from tests._oracle_pool import switch_many

pytestmark = pytest.mark.gpu

U64_MAX = (1 << 64) - 1


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.close()


def gpu_switch(eng, recs, cur, horizon):
    from paper_conf_icpp_hulww24_b200 import as_u64
    arr = np.ascontiguousarray(np.asarray(recs, dtype=np.uint8).reshape(-1, 16))
    out = eng.switch_rewards(torch.from_numpy(arr), cur, horizon)
    torch.cuda.synchronize()
    cols = [[int(x) for x in as_u64(out[k])] for k in ("time", "refill", "migrate", "reward")]
    return list(zip(*cols))


def _recs(L, N, n, seed, p=0.6):
    return W.sample_records(L, N, n, seed, random_placement_p=p)


@pytest.mark.parametrize("seed", range(6))
def test_random_small(eng, seed):
    """Random profiles and states (independent per-worker f/b, asymmetric links, zeros), random
    proposals with replicas and arbitrary placement, invalid records, the current partition itself."""
    rng = np.random.default_rng(900 + seed)
    for it in range(3):
        L = int(rng.integers(2, 30))
        N = int(rng.integers(1, 9))
        prof = W.random_profile(L, rng, f_max=1000, bytes_max=10**6)
        st = W.random_state_small(prof, N, rng, tau_max=10**4)
        eng.load(prof, st)
        recs = _recs(L, N, 300, seed * 10 + it)
        recs = np.concatenate([recs, W.corrupt_records(recs[:60], L, N, seed)])
        cur = bytes(recs[int(rng.integers(0, 300))])
        recs = np.concatenate([recs, np.frombuffer(cur, dtype=np.uint8)[None, :]])
        h = int(rng.choice([1, 3, 1000]))
        assert gpu_switch(eng, recs, cur, h) == switch_many(prof, st, [bytes(r) for r in recs], cur, h)


@pytest.mark.parametrize("name", ["vgg16", "resnet50", "gnmt16", "bert24"])
def test_paper_profiles(eng, name):
    prof = W.profile(name)
    rng = np.random.default_rng(7)
    st = W.random_state(prof, 8, rng, free_link_p=0.1)
    eng.load(prof, st)
    recs = _recs(prof.L, 8, 400, 31)
    cur = bytes(recs[5])
    assert gpu_switch(eng, recs, cur, 16) == switch_many(prof, st, [bytes(r) for r in recs], cur, 16)


def test_gpt96_from_even_split(eng):
    """The 96-layer config: proposals near the even split (its two-worker neighbourhood) and random
    8-stage records, versus the even split as the current partition."""
    prof, st = W.gpt96(), W.gpt_state("b")
    eng.load(prof, st)
    even = W.contiguous_record(96, [11, 23, 35, 47, 59, 71, 83], [1] * 8)
    nb = eng.neighbourhood(even).cpu().numpy()
    rng = np.random.default_rng(3)
    pick = nb[rng.choice(len(nb), size=min(150, len(nb)), replace=False)]
    recs = np.concatenate([pick, _recs(96, 8, 150, 77, p=0.3)])
    assert gpu_switch(eng, recs, even, 100) == switch_many(prof, st, [bytes(r) for r in recs], even, 100)


def test_outputs_optional_and_errors(eng):
    from paper_conf_icpp_hulww24_b200 import AutopipeError, as_u64
    from paper_conf_icpp_hulww24_b200._lib import AUTOPIPE_E_INVAL, AUTOPIPE_E_OVERFLOW
    prof, st = W.vgg16(), W.vgg_state()
    eng.load(prof, st)
    recs = torch.from_numpy(_recs(prof.L, 8, 200, 5))
    cur = bytes(recs[0].numpy())
    full = eng.switch_rewards(recs, cur, 4)
    only = eng.switch_rewards(recs, cur, 4, outputs=())
    assert set(only) == {"reward"}
    assert torch.equal(full["reward"], only["reward"])
    # the reward agrees with the eval kernel's T where nothing switches and exceeds it elsewhere
    t = as_u64(eng.eval_partitions(recs))
    assert np.array_equal(np.asarray(as_u64(full["time"])), np.asarray(t))
    with pytest.raises(AutopipeError) as ex:
        eng.switch_rewards(recs, cur, 0)
    assert ex.value.code == AUTOPIPE_E_INVAL
    with pytest.raises(AutopipeError) as ex:
        eng.switch_rewards(recs, W.encode(0, [], [0] * 8), 1)
    assert ex.value.code == AUTOPIPE_E_INVAL
    # a state whose modelled sums reach 2^52 ns is refused (its startup times could wrap)
    big = W.State([[1 << 50] * prof.L] * 8, [[1 << 50] * prof.L] * 8, st.tau)
    eng.set_state(big.f, big.b, big.tau)
    with pytest.raises(AutopipeError) as ex:
        eng.switch_rewards(recs, cur, 1)
    assert ex.value.code == AUTOPIPE_E_OVERFLOW


def test_device_state(eng):
    """A state given in device memory: same numbers as the host state."""
    prof, st = W.resnet50(), W.rollout_state(W.resnet50(), 1)
    eng.load(prof, st)
    recs = _recs(prof.L, st.N, 500, 9)
    cur = bytes(recs[1])
    ref = gpu_switch(eng, recs, cur, 8)
    dev = lambda a: torch.tensor(a, dtype=torch.int64, device="cuda")
    eng.set_state_device(dev(st.f), dev(st.b), dev(st.tau))
    assert gpu_switch(eng, recs, cur, 8) == ref
