#!/usr/bin/env python
"""Row e, cross-shard bound: device time per shard of the 96-layer search split G ways with
cost-balanced shards (what each of G GPUs would run), one shard at a time on one GPU — without the
bound (each shard seeds itself) and with it (seed-only call per shard, the seeds' minimum as every
shard's starting theta). Prints one JSON object: per G and state, the slowest shard's search time,
the slowest seed-only call, and both results (they must agree)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__  # noqa: E402

__graft_entry__.build()
import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine, reduce_results, result_from_bytes  # noqa: E402
from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds  # noqa: E402

eng = Engine(0)
eng.set_timing(True)
dev = torch.device("cuda", 0)
out = {}


def timed(fn, reps=3):
    best = None
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        r = fn()
        b.record()
        torch.cuda.synchronize()
        t = a.elapsed_time(b)
        best = t if best is None else min(best, t)
    return best, r


for kind in ("a-nvlink", "b"):
    eng.load(W.gpt96(), W.gpt_state(kind))
    for G in (2, 4, 8):
        bd = balanced_bounds(96, 8, 8, 8, 0, G)
        plain, seeds, seed_ms, res_plain = [], [], [], []
        for i in range(G):
            ms = []
            for _ in range(3):
                r = eng.search_optimum(8, 8, begin=bd[i], end=bd[i + 1])
                ms.append(eng.last_search_ms)
            plain.append(min(ms))
            res_plain.append(r)
            t, s = timed(lambda: eng.search_seed_async(8, 8, begin=bd[i], end=bd[i + 1]).clone())
            seed_ms.append(t)
            seeds.append(int(s.cpu().numpy().view(np.uint64)[0]))
        theta = torch.tensor(np.array([min(seeds)], dtype=np.uint64).view(np.int64), device=dev)
        eng.set_search_bound(theta)
        bounded, outs = [], []
        for i in range(G):
            ms = []
            for _ in range(3):
                o = eng.search_optimum_async(8, 8, begin=bd[i], end=bd[i + 1])
                torch.cuda.synchronize()
                ms.append(eng.last_search_ms)
            bounded.append(min(ms))
            outs.append(o)
        eng.set_search_bound(None)
        red = result_from_bytes(reduce_results(torch.stack(outs)))
        best = min(res_plain, key=lambda r: (r.time_ns, r.index))
        out["%s_G%d" % (kind, G)] = {
            "max_shard_ms_unbounded": max(plain), "max_shard_ms_bounded": max(bounded),
            "max_seed_call_ms": max(seed_ms), "theta": min(seeds),
            "per_shard_unbounded": [round(x, 4) for x in plain], "per_shard_bounded": [round(x, 4) for x in bounded],
            "same_optimum": (red.time_ns, red.index) == (best.time_ns, best.index),
            "optimum": [red.time_ns, red.index]}
print(json.dumps(out))
