"""Round-robin replicas (row f4): a C5 ResNet-50 record whose schedule has no periodic regime within
200,000 rounds (two near-equal cycle ratios): both the oracle and the kernel fall back to ceil(lambda)
from the one-period event graph (Bellman-Ford on integer theta) and agree."""
import numpy as np
import pytest
import torch

import workloads as W
from oracle import roundrobin as RR

pytestmark = pytest.mark.gpu

# stage 0 = layers 0..15 on worker 4, stage 1 = 16..29 on workers 0 and 3, stage 2 = 30..49 on worker 2
REC = W.encode(3, [15, 29], [1, W.IDLE, 2, 1, 0])


@pytest.mark.parametrize("mode", [{}, {"rr_defer_all": True}, {"rr_no_defer": True}])
def test_long_transient_record(mode):
    from paper_conf_icpp_hulww24_b200 import Engine, as_u64
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    eng = Engine(0)
    eng.load(prof, st)
    eng.set_schedule(4)
    eng.set_search_options(**mode)
    got = as_u64(eng.eval_partitions(torch.from_numpy(np.frombuffer(REC, dtype=np.uint8).reshape(1, 16).copy())))
    eng.close()
    assert int(got[0]) == RR.score_record(prof, st, REC) == 591221519
