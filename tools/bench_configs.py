#!/usr/bin/env python
"""Secondary measurements on the other BASELINE.json configs (1 GPU, device-timed with CUDA events):

  C1 toy       exhaustive search of the 165-candidate space
  C2 VGG-16    exhaustive search (1,184,040 candidates, replicas, heterogeneous links)
  C3 GNMT-16 / BERT-24 state trace: per state switch, set_state + full search (re-score latency)
  C5 ResNet-50 rollouts: 1M random records per step, eval and rollout (T + switch bytes)
  f1 / f2 / f3 NEXT rows: neighbourhood step, switch rewards, schedule variants (BERT-24 search, rollouts)

Used by bench.py (key "configs") and runnable on its own.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def _timed(fn, reps=5, warm=2):
    """Device time per call: `reps` calls enqueued back to back between one pair of CUDA events
    (asynchronous calls keep the GPU busy, so the host's enqueue cost is hidden as it is in a
    pipeline; calls that synchronise internally are timed with their host round trip)."""
    import torch
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


def measure(device: int = 0, rollout_records: int = 1 << 20):
    import torch
    import workloads as W
    from paper_conf_icpp_hulww24_b200 import Engine
    eng = Engine(device)
    res = {}
    # C1 / C2: exhaustive searches
    for name, prof, st, smax in (("C1_toy", W.toy(), W.toy_state(), 4), ("C2_vgg16", W.vgg16(), W.vgg_state(), 8)):
        eng.load(prof, st)
        n = eng.count_candidates(1, smax)
        ms, r = _timed(lambda: eng.search_optimum(1, smax))
        res[name] = {"candidates": n, "ms_to_optimum": ms, "evals_per_s": n / (ms / 1e3),
                     "optimum_T_ns": r.time_ns, "optimum_index": r.index, "int_path": eng.int_path}
    # C3: state traces, re-score latency per switch (state copy + state kernel + search)
    for name in ("gnmt16", "bert24"):
        prof = W.profile(name)
        eng.load_profile(prof.O, prof.G, prof.P)
        per = []
        for st in W.trace_c3(prof):
            smax = min(8, st.N)

            def step(st=st, smax=smax):
                eng.set_state(st.f, st.b, st.tau)
                return eng.search_optimum(1, smax)
            ms, r = _timed(step, reps=3, warm=1)
            n = eng.count_candidates(1, smax)
            per.append({"state": st.label, "N": st.N, "candidates": n, "ms": ms, "T_ns": r.time_ns,
                        "index": r.index})
        res["C3_" + name] = {"states": len(per), "mean_rescore_ms": sum(p["ms"] for p in per) / len(per),
                             "max_rescore_ms": max(p["ms"] for p in per), "per_state": per}
    # C5: rollouts
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    eng.load(prof, st)
    recs = torch.from_numpy(W.sample_records(prof.L, st.N, rollout_records, 1000)).cuda()
    cur = bytes(recs[0].cpu().numpy())
    out_t = torch.empty(rollout_records, dtype=torch.int64, device="cuda")
    out_s = torch.empty_like(out_t)
    ms_e, _ = _timed(lambda: eng.eval_partitions(recs, out=out_t))
    ms_r, _ = _timed(lambda: eng.rollout_rewards(recs, cur, out_t=out_t, out_sw=out_s))
    ms_s, _ = _timed(lambda: eng.switch_rewards(recs, cur, 100, outputs=(), stream=None))
    res["F2_resnet50_switch_rewards"] = {"records": rollout_records, "ms": ms_s,
                                         "records_per_s": rollout_records / (ms_s / 1e3), "horizon": 100}
    # C5 step latency: every step a new cluster state (rollout_state(step)) and a new
    # batch (seed 1000 + step, already on the device): set_state from host arrays (host overflow check,
    # H2D, state kernel) + rollout rewards, one CUDA-event pair per step around both
    import numpy as _np
    nst = 4
    states = [W.rollout_state(prof, k) for k in range(nst)]
    batches = [torch.from_numpy(W.sample_records(prof.L, states[k].N, rollout_records, 1000 + k)).cuda()
               for k in range(nst)]
    curs = [bytes(bt[0].cpu().numpy()) for bt in batches]
    step_ms = []
    for rep in range(2):
        for k in range(nst):
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            eng.set_state(states[k].f, states[k].b, states[k].tau)
            eng.rollout_rewards(batches[k], curs[k], out_t=out_t, out_sw=out_s)
            b.record()
            torch.cuda.synchronize()
            if rep:
                step_ms.append(a.elapsed_time(b))
    del batches
    eng.load(prof, st)
    res["C5_resnet50_rollout"] = {"records": rollout_records, "eval_ms": ms_e,
                                  "step_ms_set_state_plus_rollout": float(_np.mean(step_ms)),
                                  "step_states": nst,
                                  "eval_records_per_s": rollout_records / (ms_e / 1e3),
                                  "rollout_ms": ms_r, "rollout_records_per_s": rollout_records / (ms_r / 1e3),
                                  "eval_GBps_algorithmic": rollout_records * 24 / (ms_e / 1e3) / 1e9,
                                  "int_path": eng.int_path}
    # full-T scoring of the records the SURVEY's 230-op unit describes: 1M random S = 8, r = 1
    # partitions of the 96-layer profile (state C4a, 32-bit path), every T computed in full
    gp = W.gpt96()
    eng.load(gp, W.gpt_state("a-nvlink"))
    r1recs = torch.from_numpy(W.r1_records(gp.L, 8, rollout_records, 96)).cuda()
    ms_r1, _ = _timed(lambda: eng.eval_partitions(r1recs, out=out_t))
    res["C4_gpt96_r1_records"] = {"records": rollout_records, "eval_ms": ms_r1,
                                  "eval_records_per_s": rollout_records / (ms_r1 / 1e3), "int_path": eng.int_path}
    # f1: the paper's two-worker neighbourhood step and its gradual migration on
    # the 96-layer profile, heterogeneous state C4b, starting from the even split
    prof, st = W.gpt96(), W.gpt_state("b")
    eng.load(prof, st)
    even = W.contiguous_record(96, [11, 23, 35, 47, 59, 71, 83], [1] * 8)
    ms_n, r = _timed(lambda: eng.best_neighbour(even))
    import time as _t
    t0 = _t.perf_counter()
    path = eng.local_search(even, max_steps=500)
    ls_s = _t.perf_counter() - t0
    opt = eng.search_optimum(8, 8)
    res["F1_neighbourhood_gpt96_C4b"] = {"neighbours": r.evaluated, "ms_per_step": ms_n,
                                         "local_search_steps": len(path) - 1, "local_search_wall_ms": 1e3 * ls_s,
                                         "start_T_ns": path[0][0], "local_opt_T_ns": path[-1][0],
                                         "exhaustive_opt_T_ns": opt.time_ns,
                                         "local_over_exhaustive": path[-1][0] / opt.time_ns}
    # f3: schedule variants on the BERT profile the paper uses for its DAPPLE / 2BW comparison
    # (BERT-24 here), all-100 Gb/s state, M = 8 micro-batches: exhaustive search
    # of S in [1, 8], sum r <= 8 under each model; ResNet-50 rollout records scored per schedule.
    from paper_conf_icpp_hulww24_b200 import _lib as L_
    prof = W.bert24()
    st = W.trace_c3(prof)[0]
    eng.load(prof, st)
    n = eng.count_candidates(1, 8)
    f3 = {}
    for label, model in (("pipedream_ring", (L_.SCHED_PIPEDREAM, L_.SYNC_RING, 1, False)),
                         ("pipedream_ps", (L_.SCHED_PIPEDREAM, L_.SYNC_PS, 1, False)),
                         ("2bw_M8", (L_.SCHED_2BW, L_.SYNC_RING, 8, False)),
                         ("gpipe_M8_recompute", (L_.SCHED_GPIPE, L_.SYNC_RING, 8, True)),
                         ("dapple_M8", (L_.SCHED_DAPPLE, L_.SYNC_RING, 8, False)),
                         ("chimera_M8", (L_.SCHED_CHIMERA, L_.SYNC_RING, 8, False)),
                         ("pipedream_rr", (L_.SCHED_PIPEDREAM_RR, L_.SYNC_RING, 1, False))):
        eng.set_schedule(*model)
        ms, r = _timed(lambda: eng.search_optimum(1, 8), reps=3, warm=1)
        rec = r.partition
        f3[label] = {"ms_to_optimum": ms, "evals_per_s": n / (ms / 1e3), "optimum_T_ns": r.time_ns,
                     "optimum_index": r.index, "stages": rec[0],
                     "replicas": [sum(1 for w in range(8) if rec[8 + w] == s) for s in range(rec[0])]}
    eng.set_schedule()
    prof = W.resnet50()
    st = W.rollout_state(prof, 0)
    eng.load(prof, st)
    for label, model in (("rollout_2bw_M8", (L_.SCHED_2BW, L_.SYNC_PS, 8, False)),
                         ("rollout_gpipe_M8", (L_.SCHED_GPIPE, L_.SYNC_RING, 8, False)),
                         ("rollout_dapple_M8", (L_.SCHED_DAPPLE, L_.SYNC_PS, 8, False))):
        eng.set_schedule(*model)
        ms, _ = _timed(lambda: eng.eval_partitions(recs, out=out_t))
        f3[label] = {"records": rollout_records, "ms": ms, "records_per_s": rollout_records / (ms / 1e3)}
    # Chimera (reading F-6): one worker per stage, ResNet-50 one-worker-per-stage records
    import numpy as _np
    rng = _np.random.default_rng(77)
    crecs = []
    for _ in range(min(rollout_records, 1 << 16)):  # 64k distinct records, tiled to the batch size
        S_ = int(rng.integers(1, st.N + 1))
        cuts = sorted(int(x) for x in rng.choice(prof.L - 1, S_ - 1, replace=False)) if S_ > 1 else []
        sow = [W.IDLE] * 8
        for s_, w_ in enumerate(int(x) for x in rng.permutation(st.N)[:S_]):
            sow[w_] = s_
        crecs.append(W.encode(S_, cuts, sow))
    crecs = _np.frombuffer(b"".join(crecs), dtype=_np.uint8).reshape(-1, 16)
    crecs = torch.from_numpy(_np.ascontiguousarray(_np.resize(crecs, (rollout_records, 16)))).cuda()
    eng.set_schedule(L_.SCHED_CHIMERA, L_.SYNC_RING, 8, False)
    ms, _ = _timed(lambda: eng.eval_partitions(crecs, out=out_t))
    f3["rollout_chimera_M8"] = {"records": rollout_records, "ms": ms, "records_per_s": rollout_records / (ms / 1e3),
                                "records_kind": "one worker per stage (Chimera partitions)"}
    eng.set_schedule(L_.SCHED_PIPEDREAM_RR, L_.SYNC_RING, 1, False)
    ms, _ = _timed(lambda: eng.eval_partitions(recs, out=out_t))
    f3["rollout_pipedream_rr"] = {"records": rollout_records, "ms": ms, "records_per_s": rollout_records / (ms / 1e3),
                                  "row": "f4 round-robin replicas"}
    eng.set_schedule()
    res["F3_schedules_bert24_M8"] = dict(candidates=n, **f3)
    # f4: the paper's 10-GPU testbed (wide records): exhaustive S <= 10 search of VGG-16 and
    # ResNet-50 on 10 heterogeneous workers, and 1M wide rollout records (S <= 10)
    f4 = {}
    for name in ("vgg16", "resnet50"):
        prof = W.profile(name)
        st = W.testbed_state(prof, seed=10)
        eng.load(prof, st)
        n = eng.count_candidates(1, 10)
        ms, r = _timed(lambda: eng.search_optimum(1, 10), reps=3, warm=1)
        f4["search_" + name] = {"candidates": n, "ms_to_optimum": ms, "evals_per_s": n / (ms / 1e3),
                                "optimum_T_ns": r.time_ns, "stages": r.partition[0]}
    prof = W.resnet50()
    st = W.testbed_state(prof, seed=10)
    eng.load(prof, st)
    wrecs = torch.from_numpy(W.sample_records(prof.L, 10, rollout_records, 1010, s_max=10, wide=True)).cuda()
    ms, _ = _timed(lambda: eng.eval_partitions(wrecs, out=out_t))
    f4["eval_wide_resnet50"] = {"records": rollout_records, "ms": ms, "records_per_s": rollout_records / (ms / 1e3)}
    res["F4_testbed10"] = f4
    eng.close()
    return res


if __name__ == "__main__":
    import __graft_entry__
    __graft_entry__.build()
    print(json.dumps(measure()))
