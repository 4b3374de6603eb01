#!/usr/bin/env python
"""Where the time of one bench step goes at each shard size (1 GPU, CUDA events on the launch
stream): state kernel, search call (host prep + kernels + finalize + result copy), kernel-only time."""
import json
import os
import sys
import time
from math import comb

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__  # noqa: E402

__graft_entry__.build()
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402


def ev():
    e = torch.cuda.Event(enable_timing=True)
    e.record()
    return e


eng = Engine(0)
out = {}
for kind in ("a-nvlink", "b"):
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng.load(prof, st)
    d = lambda a: torch.tensor(a, dtype=torch.int64, device="cuda")
    fp, bp, tau = d(st.f), d(st.b), d(st.tau)
    total = comb(95, 7)
    for G in (1, 8):
        for r in ([0, G - 1] if G > 1 else [0]):
            lo, hi = r * total // G, (r + 1) * total // G
            rows = []
            for it in range(6):
                torch.cuda.synchronize()
                e0 = ev()
                eng.set_state_device(fp, bp, tau)
                e1 = ev()
                eng.set_timing(True)
                h0 = time.perf_counter()
                eng.search_optimum(8, 8, begin=lo, end=hi)
                h1 = time.perf_counter()
                e2 = ev()
                torch.cuda.synchronize()
                rows.append((e0.elapsed_time(e1), e1.elapsed_time(e2), eng.last_search_ms, 1e3 * (h1 - h0)))
            rows = rows[2:]
            key = "%s_G%d_r%d" % (kind, G, r)
            out[key] = {k: min(x[i] for x in rows) for i, k in
                        enumerate(("state_ms", "search_call_ms", "kernel_ms", "host_wall_ms"))}
print(json.dumps(out, indent=1))
