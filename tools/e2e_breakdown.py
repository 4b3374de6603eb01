#!/usr/bin/env python
"""Host-side cost of bench.py's e2e step (C4a): load_profile + set_state from host buffers, the
asynchronous search and the 40-byte result read, with the inputs as Python lists and as uint64 numpy
arrays; wall clock per call averaged over repetitions (the GPU work of the search itself included
in the last column)."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import __graft_entry__  # noqa: E402

__graft_entry__.build()
import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_icpp_hulww24_b200 import Engine, result_from_bytes  # noqa: E402


def main(reps=30):
    eng = Engine(0)
    prof, st = W.gpt96(), W.gpt_state("a-nvlink")
    eng.load(prof, st)
    out = {}
    arrs = {"lists": (prof.O, prof.G, prof.P, st.f, st.b, st.tau),
            "numpy": tuple(np.asarray(x, dtype=np.uint64) for x in (prof.O, prof.G, prof.P, st.f, st.b, st.tau))}
    for name, (O, G, P, f, b, tau) in arrs.items():
        for label, fn in (("load_profile", lambda: eng.load_profile(O, G, P)),
                          ("set_state", lambda: eng.set_state(f, b, tau)),
                          ("step", lambda: (eng.load_profile(O, G, P), eng.set_state(f, b, tau),
                                            result_from_bytes(eng.search_optimum_async(8, 8))))):
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for _ in range(reps):
                fn()
            torch.cuda.synchronize()
            out["%s_%s_ms" % (name, label)] = 1000 * (time.perf_counter() - t0) / reps
    print(json.dumps(out))


if __name__ == "__main__":
    main()
