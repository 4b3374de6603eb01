#!/usr/bin/env python
"""Device time of the 96-layer search per shard when the space is split G ways (what each of G GPUs
would run), measured one shard at a time on one GPU: the strong-scaling ceiling of the kernel."""
import json
import os
import sys
from math import comb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__  # noqa: E402

__graft_entry__.build()
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402

eng = Engine(0)
out = {}
for kind in ("a-nvlink", "b"):
    eng.load(W.gpt96(), W.gpt_state(kind))
    eng.set_timing(True)
    total = comb(95, 7)
    for G in (1, 2, 4, 8):
        worst = 0.0
        for r in range(G):
            lo, hi = r * total // G, (r + 1) * total // G
            eng.search_optimum(8, 8, begin=lo, end=hi)
            ms = []
            for _ in range(3):
                eng.search_optimum(8, 8, begin=lo, end=hi)
                ms.append(eng.last_search_ms)
            worst = max(worst, min(ms))
        out["%s_G%d" % (kind, G)] = {"max_shard_kernel_ms": worst, "ideal_ms": None}
    base = out["%s_G1" % kind]["max_shard_kernel_ms"]
    for G in (1, 2, 4, 8):
        out["%s_G%d" % (kind, G)]["ideal_ms"] = base / G
print(json.dumps(out))
