"""One C2 VGG-16 search and one C3 BERT-24 re-score (set_state + search), after warm-up: for an ncu
launch list of the short searches (which kernels, how long each, how many)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine  # noqa: E402

eng = Engine(0)
eng.load(W.vgg16(), W.vgg_state())
for _ in range(3):
    r = eng.search_optimum(1, 8)
prof = W.bert24()
st = W.trace_c3(prof)[0]
eng.load(prof, st)
for _ in range(3):
    eng.set_state(st.f, st.b, st.tau)
    r2 = eng.search_optimum(1, 8)
torch.cuda.synchronize()
print(r.time_ns, r2.time_ns)
