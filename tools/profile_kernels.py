#!/usr/bin/env python
"""One launch of each hot kernel, for ncu captures (not a benchmark), in this order:
C4a search (k_search_r1 u32 path), C4b search (u64 path), the 1M-record C5 ResNet-50 rollout and eval
(k_eval, narrow path), switch rewards (k_switch, f2), DAPPLE M = 8 eval (f3), the 10-GPU ResNet-50
testbed search (k_search_dfs, f4 wide), C2 VGG-16 (dense k_search_generic), round-robin replicas
(f4) on the 1M C5 records, Chimera (f3) on 64k records, and the BERT-24 round-robin search
(k_search_rr and its drain)."""
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
from paper_conf_icpp_hulww24_b200 import _lib as L_  # noqa: E402

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
eng.set_schedule(L_.SCHED_DAPPLE, 0, 8)
t3 = eng.eval_partitions(recs)
torch.cuda.synchronize()
eng.set_schedule()
tb = W.testbed_state(prof, seed=10)
eng.load(prof, tb)
r = eng.search_optimum(1, 10)
print("testbed", r.time_ns, r.index)
eng.load(W.vgg16(), W.vgg_state())
r = eng.search_optimum(1, 8)
print("vgg", r.time_ns, r.index)
eng.load(prof, st)
eng.set_schedule(L_.SCHED_PIPEDREAM_RR)
eng.eval_partitions(recs)  # round-robin replicas: k_eval + the drain of its deferred records
small = recs[: 1 << 16].contiguous()
eng.set_schedule(L_.SCHED_CHIMERA, 0, 8)
eng.eval_partitions(small)
torch.cuda.synchronize()
bert = W.bert24()
eng.load(bert, W.trace_c3(bert)[0])
eng.set_schedule(L_.SCHED_PIPEDREAM_RR)
r = eng.search_optimum(1, 8)  # k_search_rr + k_rr_drain_search
print("rr search", r.time_ns, r.index)
eng.set_schedule()
print("done")
