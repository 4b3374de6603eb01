#!/usr/bin/env python
"""Device time to the exact optimum of the exhaustive searches served by the general search kernel
(C2 VGG-16, the C3 first states, the 10-GPU testbed spaces of row f4), each checked against the
previous run's optimum if given.

  python tools/search_times.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import __graft_entry__
    __graft_entry__.build()
    import workloads as W
    from paper_conf_icpp_hulww24_b200 import Engine
    eng = Engine(0)
    cases = [("C2_vgg16", W.vgg16(), W.vgg_state(), 8),
             ("C3_gnmt16_s0", W.gnmt16(), W.trace_c3(W.gnmt16())[0], 8),
             ("C3_bert24_s0", W.bert24(), W.trace_c3(W.bert24())[0], 8),
             ("F4_vgg16_testbed", W.vgg16(), W.testbed_state(W.vgg16(), seed=10), 10),
             ("F4_resnet50_testbed", W.resnet50(), W.testbed_state(W.resnet50(), seed=10), 10)]
    res = {}
    for name, prof, st, smax in cases:
        eng.load(prof, st)
        reps = 1 if "resnet50_testbed" in name else 5
        r = eng.search_optimum(1, smax)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(reps):
            r = eng.search_optimum(1, smax)
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / reps
        res[name] = {"ms": ms, "T": r.time_ns, "index": r.index, "evaluated": r.evaluated,
                     "decided_per_s": r.evaluated / ms * 1e3}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
