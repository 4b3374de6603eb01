#!/usr/bin/env python
"""Device time of one 1M-record C5 eval batch (ResNet-50, App. B) per rollout state: 20 launches back
to back between CUDA events, per state (the state's N sets the replica mix).

  python tools/eval_states.py [states] [mode: eval|rollout|switch]
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
    nstates = int(sys.argv[1]) if len(sys.argv) > 1 else 6
    mode = sys.argv[2] if len(sys.argv) > 2 else "eval"
    eng, prof, n = Engine(0), W.resnet50(), 1 << 20
    out = []
    for step in range(nstates):
        st = W.rollout_state(prof, step)
        eng.load(prof, st)
        recs = torch.from_numpy(W.sample_records(prof.L, st.N, n, 1000 + step)).cuda()
        cur = bytes(recs[0].cpu().numpy())
        o = torch.empty(n, dtype=torch.int64, device="cuda")
        o2 = torch.empty(n, dtype=torch.int64, device="cuda")

        def call():
            if mode == "eval":
                eng.eval_partitions(recs, out=o)
            elif mode == "rollout":
                eng.rollout_rewards(recs, cur, out_t=o, out_sw=o2)
            else:
                eng.switch_rewards(recs, cur, 100)
        for _ in range(3):
            call()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(20):
            call()
        b.record()
        torch.cuda.synchronize()
        us = a.elapsed_time(b) / 20 * 1000
        out.append({"state": step, "N": st.N, "us": us, "records_per_s": n / us * 1e6})
    print(json.dumps({"mode": mode, "per_state": out, "mean_us": sum(x["us"] for x in out) / len(out)}))


if __name__ == "__main__":
    main()
