#!/usr/bin/env python
"""Throughput of the explicit-record kernels (eval / rollout) on the C5 workload (App. B):
ResNet-50, 1M random partition records per step, a fresh cluster state per step."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import __graft_entry__  # noqa: E402

__graft_entry__.build()
import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402


def run(n=1 << 20, steps=10):
    eng = Engine(0)
    prof = W.resnet50()
    res = {}
    for mode in ("eval", "rollout"):
        ms = []
        for step in range(steps + 3):
            st = W.rollout_state(prof, step)
            eng.load(prof, st)
            recs = torch.from_numpy(W.sample_records(prof.L, st.N, n, 1000 + step)).cuda()
            cur = bytes(recs[0].cpu().numpy())
            out_t = torch.empty(n, dtype=torch.int64, device="cuda")
            out_s = torch.empty(n, dtype=torch.int64, device="cuda")
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            reps = 5  # back to back: device time per batch, host enqueue hidden
            a.record()
            for _ in range(reps):
                if mode == "eval":
                    eng.eval_partitions(recs, out=out_t)
                else:
                    eng.rollout_rewards(recs, cur, out_t=out_t, out_sw=out_s)
            b.record()
            torch.cuda.synchronize()
            if step >= 3:
                ms.append(a.elapsed_time(b) / reps)
        avg = sum(ms) / len(ms)
        bytes_per = 24 if mode == "eval" else 32
        res[mode] = {"records_per_s": n / (avg / 1e3), "ms_per_batch": avg, "records": n,
                     "hbm_GBps_algorithmic": n * bytes_per / (avg / 1e3) / 1e9, "int_path": eng.int_path}
    print(json.dumps(res))


if __name__ == "__main__":
    run()
