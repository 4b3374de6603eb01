"""The bound-pruned searches of rows f3/f4 (GPipe, DAPPLE, Chimera: k_search_generic with
model_lower; round-robin replicas: k_search_rr with its deferral drain) against the oracle's minimum
over a medium enumeration (VGG-16-shaped profile, 6 heterogeneous workers, S <= 4: 21,206
candidates, every one scored by the oracle). A lower bound that were ever above the true T of the
optimum would prune it and fail here; the shard split checks the result does not depend on where
the launch's running best comes from."""
import numpy as np
import pytest

import workloads as W
from oracle import schedules as SC
from oracle.enumerate import candidates, count
from oracle.model import encode_partition
from tests._oracle_pool import chimera_many, rr_many, sched_many

pytestmark = pytest.mark.gpu
SCHED_RR, SCHED_CHIMERA = 4, 5


@pytest.fixture(scope="module")
def space():
    prof = W.vgg16()
    rng = np.random.default_rng(77)
    st = W.random_state_small(prof, 6, rng, tau_max=4000)
    recs = [encode_partition(p) for p in candidates(prof.L, 6, 1, 4, 0)]
    assert len(recs) == count(prof.L, 6, 1, 4) == 21206
    return prof, st, recs


@pytest.fixture(scope="module")
def eng():
    from paper_conf_icpp_hulww24_b200 import Engine
    e = Engine(0)
    yield e
    e.set_schedule()
    e.close()


MODELS = {
    "gpipe_M4_recompute": ((SC.GPIPE, SC.RING, 4, True), lambda p, s, r: sched_many(p, s, r, SC.GPIPE, SC.RING, 4, True)),
    "dapple_M8_ps": ((SC.DAPPLE, SC.PS, 8, False), lambda p, s, r: sched_many(p, s, r, SC.DAPPLE, SC.PS, 8, False)),
    "gpipe_M2": ((SC.GPIPE, SC.PS, 2, False), lambda p, s, r: sched_many(p, s, r, SC.GPIPE, SC.PS, 2, False)),
    "dapple_M3": ((SC.DAPPLE, SC.RING, 3, False), lambda p, s, r: sched_many(p, s, r, SC.DAPPLE, SC.RING, 3, False)),
    "dapple_M1": ((SC.DAPPLE, SC.RING, 1, False), lambda p, s, r: sched_many(p, s, r, SC.DAPPLE, SC.RING, 1, False)),
    "chimera_M6": ((SCHED_CHIMERA, 0, 6, False), lambda p, s, r: chimera_many(p, s, r, 6)),
    "roundrobin": ((SCHED_RR, 0, 1, False), lambda p, s, r: rr_many(p, s, r)),
}


@pytest.mark.parametrize("name", list(MODELS))
def test_pruned_search_medium_space(eng, space, name):
    prof, st, recs = space
    model, oracle_fn = MODELS[name]
    ts = oracle_fn(prof, st, recs)
    best = min(range(len(ts)), key=lambda i: (ts[i], i))
    eng.load(prof, st)
    eng.set_schedule(*model)
    r = eng.search_optimum(1, 4)
    mid = len(recs) // 2 + 17
    a, b = eng.search_optimum(1, 4, 0, 0, mid), eng.search_optimum(1, 4, 0, mid)
    eng.set_schedule()
    assert (r.time_ns, r.index, r.evaluated) == (ts[best], best, len(recs))
    assert min((a.time_ns, a.index), (b.time_ns, b.index)) == (ts[best], best)
    assert a.evaluated + b.evaluated == len(recs)
