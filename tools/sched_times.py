#!/usr/bin/env python
"""Device time of the slow schedule models (round-robin replicas, Chimera) on the bench workloads:
1M C5 ResNet-50 rollout records (state 0) per model, and the BERT-24 exhaustive search (S <= 8,
sum r <= 8, M = 8). Quick iteration tool; the bench line carries the same numbers under configs.F3."""
import json
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


def timed(fn, reps=3, warm=1):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        r = fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps, r


def chimera_records(L, N, n, seed=77):
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(min(n, 1 << 16)):
        S = int(rng.integers(1, N + 1))
        cuts = sorted(int(x) for x in rng.choice(L - 1, S - 1, replace=False)) if S > 1 else []
        sow = [W.IDLE] * 8
        for s, w in enumerate(int(x) for x in rng.permutation(N)[:S]):
            sow[w] = s
        out.append(W.encode(S, cuts, sow))
    a = np.frombuffer(b"".join(out), dtype=np.uint8).reshape(-1, 16)
    return torch.from_numpy(np.ascontiguousarray(np.resize(a, (n, 16)))).cuda()


def main():
    which = sys.argv[1:] or ["rr", "chimera"]
    eng = Engine(0)
    res = {}
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    eng.load(prof, st)
    n = 1 << 20
    recs = torch.from_numpy(W.sample_records(prof.L, st.N, n, 1000)).cuda()
    out = torch.empty(n, dtype=torch.int64, device="cuda")
    if "switch" in which:
        cur = bytes(recs[0].cpu().numpy())
        res["switch_1M_ms"], _ = timed(lambda: eng.switch_rewards(recs, cur, 100, outputs=()), reps=10, warm=2)
    if "flush" in which:
        for k, model in (("gpipe", (L_.SCHED_GPIPE, L_.SYNC_RING, 8, False)), ("dapple", (L_.SCHED_DAPPLE, L_.SYNC_PS, 8, False))):
            eng.set_schedule(*model)
            res[k + "_eval_1M_ms"], _ = timed(lambda: eng.eval_partitions(recs, out=out), reps=10, warm=2)
        eng.set_schedule()
    if "c5" in which:
        res["c5_eval_1M_ms"], _ = timed(lambda: eng.eval_partitions(recs, out=out), reps=20, warm=3)
    if "rr" in which or "rr_eval" in which:
        eng.set_schedule(L_.SCHED_PIPEDREAM_RR, L_.SYNC_RING, 1, False)
        res["rr_eval_1M_ms"], _ = timed(lambda: eng.eval_partitions(recs, out=out))
        eng.set_search_options(rr_no_defer=True)
        res["rr_eval_1M_no_defer_ms"], _ = timed(lambda: eng.eval_partitions(recs, out=out))
        eng.set_search_options()
    if "chimera" in which:
        crecs = chimera_records(prof.L, st.N, n)
        eng.set_schedule(L_.SCHED_CHIMERA, L_.SYNC_RING, 8, False)
        res["chimera_eval_1M_ms"], _ = timed(lambda: eng.eval_partitions(crecs, out=out))
    eng.set_schedule()
    if "r1" in which:
        gp = W.gpt96()
        eng.load(gp, W.gpt_state("a-nvlink"))
        r1 = torch.from_numpy(W.r1_records(gp.L, 8, n, 5)).cuda()
        res["gpt96_r1_eval_1M_ms"], _ = timed(lambda: eng.eval_partitions(r1, out=out), reps=20, warm=3)
    prof = W.bert24()
    eng.load(prof, W.trace_c3(prof)[0])
    for k, model in (("rr", (L_.SCHED_PIPEDREAM_RR, L_.SYNC_RING, 1, False)),
                     ("chimera", (L_.SCHED_CHIMERA, L_.SYNC_RING, 8, False)),
                     ("gpipe", (L_.SCHED_GPIPE, L_.SYNC_RING, 8, True)),
                     ("dapple", (L_.SCHED_DAPPLE, L_.SYNC_RING, 8, False))):
        if k in which:
            eng.set_schedule(*model)
            ms, r = timed(lambda: eng.search_optimum(1, 8), reps=2)
            res[k + "_search_bert24_ms"] = ms
            res[k + "_search_bert24_T"] = r.time_ns
    eng.close()
    print(json.dumps(res))


if __name__ == "__main__":
    main()
