import os, sys
from math import comb
sys.path.insert(0, os.getcwd())
import workloads as W
from paper_conf_icpp_hulww24_b200 import Engine
eng = Engine(0)
total = comb(95, 7)
for kind in ("a-nvlink", "b"):
    eng.load(W.gpt96(), W.gpt_state(kind))
    print(kind, "G1", flush=True)
    eng.search_optimum(8, 8)
    print(kind, "G8", flush=True)
    for r in range(8):
        eng.search_optimum(8, 8, begin=r * total // 8, end=(r + 1) * total // 8)
