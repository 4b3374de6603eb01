#!/usr/bin/env python
"""Kernel time of every shard of the 96-layer space split G ways, for the state(s) given; one JSON
line. Tuning knobs come from the environment (AUTOPIPE_R1_*), so run one process per setting."""
import json
import os
import sys
from math import comb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402


def shard_times(eng, G, bounds=None, reps=3):
    total = comb(95, 7)
    bounds = bounds or [r * total // G for r in range(G)] + [total]
    out = []
    for r in range(G):
        lo, hi = bounds[r], bounds[r + 1]
        eng.search_optimum(8, 8, begin=lo, end=hi)
        ms = []
        for _ in range(reps):
            eng.search_optimum(8, 8, begin=lo, end=hi)
            ms.append(eng.last_search_ms)
        out.append(round(min(ms), 4))
    return out


if __name__ == "__main__":
    eng = Engine(0)
    eng.set_timing(True)
    res = {"env": {k: v for k, v in os.environ.items() if k.startswith("AUTOPIPE_")}}
    for kind in sys.argv[1:] or ["a-nvlink"]:
        eng.load(W.gpt96(), W.gpt_state(kind))
        from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
        for G in (1, 2, 4, 8):
            t = shard_times(eng, G)
            res["%s_G%d" % (kind, G)] = {"max": max(t), "sum": round(sum(t), 4), "shards": t}
            t = shard_times(eng, G, balanced_bounds(96, 8, 8, 8, 0, G))
            res["%s_G%d_balanced" % (kind, G)] = {"max": max(t), "sum": round(sum(t), 4), "shards": t}
    print(json.dumps(res))
