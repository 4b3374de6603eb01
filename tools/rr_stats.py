#!/usr/bin/env python
"""Round-robin replicas (row f4) diagnostics: how many rounds the kernel simulates per record before
its period is pinned, and how many records need the event-graph Bellman-Ford, on the 1M C5 ResNet-50
rollout records (state 0), every record in its own thread (no deferral). Builds the -DRR_STATS=1
variant of k_eval (the output word then holds rounds | not-pinned << 32 instead of T)."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

# the regular objects the variant links against (a subprocess: build() imports the package)
subprocess.run([sys.executable, "-c", "import __graft_entry__ as g; g.build()"], check=True, cwd=ROOT)
# argv: [variant name] [extra nvcc flags] (default: rrstats, -DRR_STATS=1)
NAME = sys.argv[1] if len(sys.argv) > 1 else "rrstats"
FLAGS = sys.argv[2] if len(sys.argv) > 2 else "-DRR_STATS=1"
N_REC = int(os.environ.get("RR_STATS_N", 1 << 20))
subprocess.run(["bash", os.path.join(ROOT, "tools", "build_variants.sh"), "%s=%s" % (NAME, FLAGS)], check=True,
               env=dict(os.environ, TUS="k_eval"))
os.environ["AUTOPIPE_LIB"] = os.path.join(ROOT, "paper_conf_icpp_hulww24_b200", "libautopipe_%s.so" % NAME)
import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine, as_u64  # noqa: E402
from paper_conf_icpp_hulww24_b200 import _lib as L_  # noqa: E402

eng = Engine(0)
prof = W.resnet50()
st = W.rollout_state(prof, 0)
eng.load(prof, st)
n = 1 << 20
recs = torch.from_numpy(W.sample_records(prof.L, st.N, n, 1000)[:N_REC].copy()).cuda()
eng.set_schedule(L_.SCHED_PIPEDREAM_RR, L_.SYNC_RING, 1, False)
eng.set_search_options(rr_no_defer=True)
v = as_u64(eng.eval_partitions(recs)).astype(np.uint64)
valid = v != np.uint64(2**64 - 1)
v = v[valid]
rounds = (v & np.uint64(0xFFFFFFFF)).astype(np.int64)
fb = ((v >> np.uint64(32)) & np.uint64(1)).astype(bool)
print("records scored", int(valid.sum()), "fallbacks", int(fb.sum()))
qs = [50, 90, 99, 99.9, 99.99, 100]
print("rounds percentiles", dict(zip(qs, np.percentile(rounds, qs).tolist())))
print("sum of rounds", int(rounds.sum()), "fallback rounds share", float(rounds[fb].sum() / max(1, rounds.sum())))
hist = np.histogram(rounds, bins=[0, 8, 16, 32, 64, 128, 256, 512, 1024, 2048, 4096, 1 << 20])
print("histogram", list(zip(hist[1][:-1].tolist(), hist[0].tolist())))
# the same records scored one per launch, against the batch
few = recs[:16].contiguous()
vb = as_u64(eng.eval_partitions(few)).astype(np.uint64)
for i in range(16):
    v1 = as_u64(eng.eval_partitions(few[i:i + 1].contiguous())).astype(np.uint64)[0]
    print(i, "batch", int(vb[i] & np.uint64(0xFFFFFFFF)), int(vb[i] >> np.uint64(32)),
          "single", int(v1 & np.uint64(0xFFFFFFFF)), int(v1 >> np.uint64(32)))
