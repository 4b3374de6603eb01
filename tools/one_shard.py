import os, sys
from math import comb
sys.path.insert(0, os.getcwd())
import workloads as W
from paper_conf_icpp_hulww24_b200 import Engine
eng = Engine(0); eng.set_timing(True)
kind = sys.argv[1] if len(sys.argv) > 1 else "b"
G = int(sys.argv[2]) if len(sys.argv) > 2 else 8
r = int(sys.argv[3]) if len(sys.argv) > 3 else 0
eng.load(W.gpt96(), W.gpt_state(kind))
total = comb(95, 7)
for _ in range(3):
    res = eng.search_optimum(8, 8, begin=r * total // G, end=(r + 1) * total // G)
print(kind, G, r, res.time_ns, res.index, eng.last_search_ms)
