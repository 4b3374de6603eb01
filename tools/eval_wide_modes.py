#!/usr/bin/env python
"""Device time of 1M wide ResNet-50 records (10 workers, S <= 10; row f4) under each schedule of
row f3 (PipeDream, 2BW, GPipe + recompute, DAPPLE; M = 8), one JSON line."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402

eng = Engine(0)
prof = W.resnet50()
st = W.testbed_state(prof, seed=10)
eng.load(prof, st)
n = 1 << 20
recs = torch.from_numpy(W.sample_records(prof.L, 10, n, 1010, s_max=10, wide=True)).cuda()
out_t = torch.empty(n, dtype=torch.int64, device="cuda")
res = {}
for name, model in (("pipedream", (0, 0, 1, False)), ("2bw", (1, 0, 8, False)),
                    ("gpipe_recompute", (2, 0, 8, True)), ("dapple", (3, 0, 8, False))):
    eng.set_schedule(*model)
    ms = []
    for i in range(8):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        eng.eval_partitions(recs, out=out_t)
        b.record()
        torch.cuda.synchronize()
        if i >= 3:
            ms.append(a.elapsed_time(b))
    res[name] = {"ms": min(ms), "records_per_s": n / (min(ms) / 1e3), "checksum": int(out_t.sum().item())}
eng.set_schedule()
print(json.dumps(res))
