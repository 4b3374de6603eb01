import os, sys
from math import comb
sys.path.insert(0, os.getcwd())
import workloads as W
from paper_conf_icpp_hulww24_b200 import Engine
from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds
eng = Engine(0); eng.set_timing(True)
eng.load(W.gpt96(), W.gpt_state("a-nvlink"))
for G in (1, 8):
    b = balanced_bounds(96, 8, 8, 8, 0, G)
    for _ in range(2):
        eng.search_optimum(8, 8, begin=b[0], end=b[1])
        print("G", G, "ms", eng.last_search_ms, flush=True)
