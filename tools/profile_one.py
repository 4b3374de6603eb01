#!/usr/bin/env python
"""One launch of a chosen kernel workload, for source-level ncu captures (not a benchmark).

  python tools/profile_one.py c5_eval | c5_rollout | c5_switch | c5_dapple | c5_gpipe | wide_dapple |
                              vgg_search | testbed_search | c4a | c4b
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import __graft_entry__  # noqa: E402

__graft_entry__.build()
import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402


def main(what):
    eng = Engine(0)
    if what.startswith("c5") or what.startswith("wide"):
        prof = W.resnet50()
        if what.startswith("wide"):
            st = W.testbed_state(prof, seed=10)
            recs = torch.from_numpy(W.sample_records(prof.L, 10, 1 << 20, 1010, s_max=10, wide=True)).cuda()
        else:
            st = W.rollout_state(prof, 0)
            recs = torch.from_numpy(W.sample_records(prof.L, st.N, 1 << 20, 1000)).cuda()
        eng.load(prof, st)
        cur = bytes(recs[0].cpu().numpy())
        if what.endswith("dapple"):
            eng.set_schedule(3, 0, 8)
        elif what.endswith("_rr"):
            eng.set_schedule(4)
        elif what.endswith("chimera"):
            eng.set_schedule(5, 0, 8)
        elif what.endswith("gpipe"):
            eng.set_schedule(2, 0, 8, True)
        if what == "c5_rollout":
            eng.rollout_rewards(recs, cur)
        elif what == "c5_switch":
            eng.switch_rewards(recs, cur, 100)
        else:
            eng.eval_partitions(recs)
    elif what == "c4_r1_records":
        gp = W.gpt96()
        eng.load(gp, W.gpt_state("a-nvlink"))
        eng.eval_partitions(torch.from_numpy(W.r1_records(gp.L, 8, 1 << 20, 96)).cuda())
    elif what == "vgg_search":
        eng.load(W.vgg16(), W.vgg_state())
        eng.search_optimum(1, 8)
    elif what == "testbed_resnet":
        prof = W.resnet50()
        eng.load(prof, W.testbed_state(prof, seed=10))
        eng.search_optimum(1, 10)
    elif what == "testbed_search":
        prof = W.vgg16()
        eng.load(prof, W.testbed_state(prof, seed=10))
        eng.search_optimum(1, 10)
    else:
        eng.load(W.gpt96(), W.gpt_state("a-nvlink" if what == "c4a" else "b"))
        eng.search_optimum(8, 8)
    torch.cuda.synchronize()
    eng.close()


if __name__ == "__main__":
    main(sys.argv[1])
