"""Parity at the bench's full sizes, in the bench's launch configuration (task ③: "at BASELINE.json's
full sizes ... on sampled outputs the oracle can compute one by one"): the 1M-record C5 ResNet-50
rollout batch of configs[4] (workloads.sample_records(50, N, 2^20, 1000), rollout state 0) scored in
one launch per model exactly as bench.py / tools/bench_configs.py time it — PipeDream eval and rollout
(T + switch bytes), the switch rewards (row f2), DAPPLE with M = 8 (row f3) and round-robin replicas
(row f4, with the deferral drain) — then a seeded sample of outputs checked one by one against the
oracle: the first and last chunk of the batch, every warp-chunk boundary in a stretch, and random
positions."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import schedules as SC
from tests._oracle_pool import rollout_many, rr_many, sched_many, switch_many

pytestmark = pytest.mark.gpu
N_REC = 1 << 20


@pytest.fixture(scope="module")
def c5():
    from paper_conf_icpp_hulww24_b200 import Engine
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    recs = W.sample_records(prof.L, st.N, N_REC, 1000)
    rng = np.random.default_rng(4242)
    idx = set(range(0, 300)) | set(range(N_REC - 300, N_REC))
    idx |= {c * 256 + d for c in range(1000, 1040) for d in (-1, 0, 1, 255)}  # 256-record chunk edges
    idx |= set(int(x) for x in rng.integers(0, N_REC, 900))
    idx = sorted(i for i in idx if 0 <= i < N_REC)
    eng = Engine(0)
    eng.load(prof, st)
    yield eng, prof, st, recs, idx
    eng.set_schedule()
    eng.close()


def _u64(t):
    from paper_conf_icpp_hulww24_b200 import as_u64
    return as_u64(t)


def test_c5_eval_and_rollout(c5):
    eng, prof, st, recs, idx = c5
    g = torch.from_numpy(recs).cuda()
    t = _u64(eng.eval_partitions(g))
    cur = bytes(recs[0])
    rt, rs = eng.rollout_rewards(g, cur)
    rt, rs = _u64(rt), _u64(rs)
    torch.cuda.synchronize()
    ot, osw = rollout_many(prof, st, [bytes(recs[i]) for i in idx], cur)
    assert [int(t[i]) for i in idx] == ot
    assert [int(rt[i]) for i in idx] == ot
    assert [int(rs[i]) for i in idx] == osw


def test_c5_switch_rewards(c5):
    eng, prof, st, recs, idx = c5
    cur = bytes(recs[7])
    out = eng.switch_rewards(torch.from_numpy(recs).cuda(), cur, 100, outputs=("time", "refill", "migrate"))
    got = {k: _u64(v) for k, v in out.items()}
    want = switch_many(prof, st, [bytes(recs[i]) for i in idx], cur, 100)
    for j, i in enumerate(idx):
        assert (int(got["time"][i]), int(got["refill"][i]), int(got["migrate"][i]), int(got["reward"][i])) == \
            tuple(want[j])


def test_c5_dapple_m8(c5):
    eng, prof, st, recs, idx = c5
    eng.set_schedule(SC.DAPPLE, SC.RING, 8, False)
    t = _u64(eng.eval_partitions(torch.from_numpy(recs).cuda()))
    eng.set_schedule()
    assert [int(t[i]) for i in idx] == sched_many(prof, st, [bytes(recs[i]) for i in idx], SC.DAPPLE, SC.RING, 8, False)


def test_c5_round_robin(c5):
    eng, prof, st, recs, idx = c5
    eng.set_schedule(4)
    t = _u64(eng.eval_partitions(torch.from_numpy(recs).cuda()))
    eng.set_schedule()
    assert [int(t[i]) for i in idx] == rr_many(prof, st, [bytes(recs[i]) for i in idx])


def test_testbed_wide_records_full_batch():
    """configs F4: 1M 32-byte wide records (S <= 10) on the 10-worker testbed state, PipeDream and
    GPipe + recompute (M = 8), sampled against the oracle."""
    from paper_conf_icpp_hulww24_b200 import Engine
    from tests._oracle_pool import score_many
    prof = W.resnet50()
    st = W.testbed_state(prof, seed=10)
    recs = W.sample_records(prof.L, 10, N_REC, 1010, s_max=10, wide=True)
    rng = np.random.default_rng(99)
    idx = sorted(set(range(0, 200)) | set(range(N_REC - 200, N_REC)) | set(int(x) for x in rng.integers(0, N_REC, 600)))
    eng = Engine(0)
    eng.load(prof, st)
    g = torch.from_numpy(recs).cuda()
    t = _u64(eng.eval_partitions(g))
    eng.set_schedule(SC.GPIPE, SC.RING, 8, True)
    tg = _u64(eng.eval_partitions(g))
    eng.set_schedule()
    eng.close()
    sub = [bytes(recs[i]) for i in idx]
    assert [int(t[i]) for i in idx] == score_many(prof, st, sub)
    assert [int(tg[i]) for i in idx] == sched_many(prof, st, sub, SC.GPIPE, SC.RING, 8, True)
