"""ORACLE — test infrastructure only.

A plain, slow CPU implementation of the AutoPipe partition cost model (SPEC.md, derived from
PAPER.md Table 1 at 788-805, Observation 2 at 486-519, Observation 3 and Fig. 2 at 521-580, and the
1F1B schedule at 253-278). Exact integer / Fraction arithmetic, pure Python.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl
reference`` legs may import anything in this package. The product path
(``paper_conf_icpp_hulww24_b200``, the C-ABI library and its kernels) never imports, links or
executes it, and this package never imports the product path. The only code both sides share is
the input generator module ``workloads`` (no cost-model arithmetic).

Modules
  model       record parsing/validity, per-op durations, transfers, all-reduce (SPEC §2-3)
  sim         event-by-event simulation of the static 1F1B schedule + exact periodicity -> lambda
  enumerate   the search index order (SPEC §5) by definition, rank/unrank
  search      brute-force search (min over the enumeration, first minimum wins)
  param_dp    parametric DP: exact search optimum + lexicographically-first argmin
  cycle_ratio max cycle ratio of the explicit timed event graph (cross-check of sim)
  rollout     rollout reward = T_ns + switch bytes (SPEC §6)
  neighbourhood  the two-worker neighbourhood by definition (NEXT f1)
  switching   switching cost as time: startup refill + weight migration, amortised reward (NEXT f2)
  schedules   schedule variants (2BW, GPipe, DAPPLE) and the sharded parameter server (NEXT f3)

Parity status: every function here is pinned by tests/test_oracle_*.py (worked examples of the
paper, closed forms, invariants, textbook reductions, brute force). None is "parity unpinned".
"""
