#!/usr/bin/env python
"""One launch of each hot kernel, for ncu captures (not a benchmark):
C4a search (u32 path), C4b search (u64 path), one 1M-record rollout batch (ResNet-50, App. B C5),
and one 1M-record switch-reward batch (NEXT row f2)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import __graft_entry__  # noqa: E402

__graft_entry__.build()
import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402

eng = Engine(0)
for kind in ("a-nvlink", "b"):
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load(prof, st)
    r = eng.search_optimum(8, 8)
    print(kind, r.time_ns, r.index, r.evaluated, eng.int_path)
prof = W.resnet50()
st = W.rollout_state(prof, 0)
eng.load(prof, st)
recs = torch.from_numpy(W.sample_records(prof.L, st.N, 1 << 20, 1000)).cuda()
t, sw = eng.rollout_rewards(recs, bytes(recs[0].cpu().numpy()))
t2 = eng.eval_partitions(recs)
torch.cuda.synchronize()
print("rollout", int((t == t2).all()))
out = eng.switch_rewards(recs, bytes(recs[0].cpu().numpy()), 100)
torch.cuda.synchronize()
print("switch", int(out["reward"].shape[0]))
# NEXT row f3: the same records under the DAPPLE schedule (flushed iteration, M = 8)
eng.set_schedule(3, 0, 8)
t3 = eng.eval_partitions(recs)
torch.cuda.synchronize()
eng.set_schedule()
print("dapple", int(t3.shape[0]))
# C2 VGG-16: the generic search kernel (replicas, heterogeneous links)
eng.load(W.vgg16(), W.vgg_state())
r = eng.search_optimum(1, 8)
print("vgg", r.time_ns, r.index)
