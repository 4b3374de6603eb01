#!/usr/bin/env python
"""Per-rank device time of bench.py's step (set_state_device + the shard's asynchronous search, L2
flushed between steps) for every rank of G = 1, 2, 4, 8, run one shard at a time on one GPU: the
strong-scaling ceiling of the step before the NCCL min-loc (which one GPU cannot run with G ranks).
Prints one JSON object: per G the per-rank ms and the max over ranks."""
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
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402
from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds  # noqa: E402


def main(kind="a-nvlink", steps=10, warm=3):
    dev = torch.device("cuda", 0)
    prof, st = W.gpt96(), W.gpt_state(kind)
    eng = Engine(0)
    eng.load_profile(prof.O, prof.G, prof.P)
    d_fp = torch.tensor(np.asarray(st.f, dtype=np.uint64).view(np.int64), device=dev)
    d_bp = torch.tensor(np.asarray(st.b, dtype=np.uint64).view(np.int64), device=dev)
    d_tau = torch.tensor(np.asarray(st.tau, dtype=np.uint64).view(np.int64), device=dev)
    eng.set_state(st.f, st.b, st.tau)  # the host classifies the integer path (the shard cost model's)
    path = eng.int_path
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream(dev)
    out = {"state": kind, "int_path": path}
    for G in (1, 2, 4, 8):
        b = balanced_bounds(96, 8, 8, 8, 0, G, path)
        per = []
        for r in range(G):
            for _ in range(warm):
                eng.set_state_device(d_fp, d_bp, d_tau)
                eng.search_optimum_async(8, 8, 0, b[r], b[r + 1])
            torch.cuda.synchronize()
            tot = 0.0
            for k in range(steps):
                flush.fill_(k)
                a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                eng.set_state_device(d_fp, d_bp, d_tau)
                eng.search_optimum_async(8, 8, 0, b[r], b[r + 1])
                z.record(stream)
                torch.cuda.synchronize()
                tot += a.elapsed_time(z)
            per.append(tot / steps)
        out[str(G)] = {"per_rank_ms": per, "max_ms": max(per)}
    print(json.dumps(out))


if __name__ == "__main__":
    main(*(sys.argv[1:2] or ["a-nvlink"]))
