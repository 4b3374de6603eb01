#!/usr/bin/env python
"""Benchmark of the AutoPipe cost-model hot path on B200 (contract: see DESIGN.md §Measurement).

One step = one pass of the whole hot path over the headline workload of BASELINE.json: the
96-layer, 8-stage exhaustive search (C(95,7) = 11,050,084,695 candidate partitions):
  a1/a2  state ingest (prefix sums, link tables) from device-resident inputs,
  a3-a8  unranking + enumeration + exact decision per candidate + argmin,
  e      the NCCL min-loc across ranks (N > 1; each rank scans 1/N of the index space).
`value` = candidates decided per second over all ranks (device time, max over ranks);
`ms_per_step` = time to the exact optimum. `e2e` = the same step through the public API from host
buffers (load_profile + set_state + search, result back on the host), wall clock, max over ranks.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--state a-nvlink|a-100g|b] [--impl ours|reference]
Under torchrun, one process per GPU (RANK/LOCAL_RANK/WORLD_SIZE from the environment).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time
from math import comb

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "partition evals/sec at 1/2/4/8 B200; time-to-exact-optimum, 96-layer 8-stage"
UNIT = "evals/s"
S_STAGES = 8
TOTAL = comb(95, 7)
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
INT_PEAK_PATH = os.path.join(ROOT, "profiles", "int_peak.json")
TRAFFIC_PATH = os.path.join(ROOT, "profiles", "round2_traffic.json")
KERNELS_PATH = os.path.join(ROOT, "profiles", "round2_kernels_full.txt")


def ncu_kernel_metrics(prefix: str):
    """Issue-slot and ALU-pipe use of the first kernel whose name starts with `prefix` in the committed
    ncu --set full summary (a capture of the same kernel on this tree; not measured by this run)."""
    want = {"smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
            "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active": "alu_pipe_active_pct",
            "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct"}
    out, inside = {}, False
    try:
        with open(KERNELS_PATH) as fh:
            for line in fh:
                if line.startswith("kernel:"):
                    if inside:
                        break
                    inside = line[len("kernel: void ap::"):].startswith(prefix) or \
                        line[len("kernel: void "):].startswith(prefix)
                    continue
                if inside:
                    parts = line.split()
                    if parts and parts[0] in want:
                        out[want[parts[0]]] = float(parts[1])
    except OSError:
        return None
    if not out:
        return None
    out["source"] = "profiles/round2_kernels_full.txt (ncu --set full, committed capture)"
    return out
# Algorithmic integer ops per candidate: the incremental full-T evaluation of an
# S = 8, r = 1 candidate under the lexicographic successor is 85 ops on the 32-bit path (x2 on the
# 64-bit path). The hot kernel only DECIDES "T <= theta" per candidate (exact T on the rare path), so
# measured against this unit its fraction exceeds 1: reported, flagged, not capped.
OPS_PER_CANDIDATE = {32: 85, 64: 170}
# full-T scoring of random records (rollouts): 230 int ops + 24 B per record (the
# S = 8, r = 1 figure, applied to every record of the C5 mix)
ROLLOUT_OPS, ROLLOUT_BYTES = 230, 24


def env_int(name, default):
    try:
        return int(os.environ.get(name, default))
    except ValueError:
        return default


def cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as fh:
            for line in fh:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


# ------------------------------------------------------------------------------------------------
# clocks during the timed region (pynvml), per the profiling recipe's clocks line
# ------------------------------------------------------------------------------------------------
REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
           0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
           0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}


class ClockSampler:
    def __init__(self, index: int, period_s: float = 0.02):
        self.samples, self.reasons, self.max_mhz = [], 0, None
        self.period = period_s
        self._stop = threading.Event()
        self._th = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        nv = self.nv
        get_r = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
            getattr(nv, "nvmlDeviceGetCurrentClocksThrottleReasons")
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                self.reasons |= int(get_r(self.h))
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.nv is not None:
            self._th = threading.Thread(target=self._run, daemon=True)
            self._th.start()
        return self

    def __exit__(self, *a):
        if self._th is not None:
            self._stop.set()
            self._th.join()

    def summary(self):
        if self.nv is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvml unavailable"]}
        names = [v for k, v in REASONS.items() if self.reasons & k and k != 0x1]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples)}


# ------------------------------------------------------------------------------------------------
# CPU baseline: the oracle, as it stands, on the host cores
# ------------------------------------------------------------------------------------------------
_PS = {}


def _oracle_init(kind):
    import workloads as W
    _PS["prof"] = W.gpt96()
    _PS["st"] = W.gpt_state(kind)


def _oracle_score(rec: bytes) -> int:
    from oracle.sim import score_record
    return score_record(_PS["prof"], _PS["st"], rec)


def oracle_sample(kind: str, n: int, seed: int):
    import numpy as np
    from oracle.enumerate import decode
    from oracle.model import encode_partition
    rng = np.random.default_rng(seed)
    return [encode_partition(decode(96, 8, 8, 8, 0, int(i))) for i in rng.integers(0, TOTAL, size=n)]


def oracle_throughput(kind: str, target_s: float = 12.0, seed: int = 12345):
    """Score a bounded random sample of the 96-layer space with the oracle on every host core."""
    import multiprocessing as mp
    ncore = cores()
    _oracle_init(kind)
    probe = oracle_sample(kind, 16, seed + 1)
    t0 = time.perf_counter()
    for r in probe:
        _oracle_score(r)
    per = (time.perf_counter() - t0) / len(probe)  # s per candidate per core
    n = max(ncore * 4, int(target_s / per * ncore))
    recs = oracle_sample(kind, n, seed)
    t0 = time.perf_counter()
    with mp.get_context("fork").Pool(ncore, initializer=_oracle_init, initargs=(kind,)) as pool:
        pool.map(_oracle_score, recs, chunksize=max(1, n // (ncore * 8)))
    dt = time.perf_counter() - t0
    return n / dt, n, dt, ncore


def param_dp_time(kind: str):
    import workloads as W
    from oracle.param_dp import optimum
    prof, st = W.gpt96(), W.gpt_state(kind)
    t0 = time.perf_counter()
    T, idx, _ = optimum(prof, st, S_STAGES, S_STAGES)
    return time.perf_counter() - t0, T, idx


def run_reference(args, rank: int, world: int):
    """--impl reference: the oracle timed on the host cores, on this arm's workload and metric."""
    if rank != 0:
        return
    import multiprocessing as mp
    ncore = cores()
    per_step = max(ncore * 600, args.ref_sample)  # ~1-2 s of oracle work per step (pool overhead amortised)
    _oracle_init(args.state)
    pool = mp.get_context("fork").Pool(ncore, initializer=_oracle_init, initargs=(args.state,))
    times = []
    for step in range(args.warmup + args.steps):
        recs = oracle_sample(args.state, per_step, 5000 + step)
        t0 = time.perf_counter()
        pool.map(_oracle_score, recs, chunksize=max(1, per_step // (ncore * 8)))
        if step >= args.warmup:
            times.append(time.perf_counter() - t0)
    pool.close()
    total_s = sum(times)
    value = per_step * args.steps / total_s
    sample = "%d random candidates of the C(95,7) space per step (seeded), oracle event simulation" % per_step
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * total_s / args.steps,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int (python)",
        "data": "synthetic", "config": config_block(args, world),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": ncore, "kind": "oracle",
                         "sample": sample, "cpu": cpu_model()},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def config_block(args, world):
    return {"workload": "96-layer transformer profile (GPT-3 shaped, App. B.6), 8 stages, exhaustive "
                        "C(95,7) cut sets; state %s" % args.state,
            "layers": 96, "stages": S_STAGES, "candidates": TOTAL, "state": args.state,
            "parallelism": "index-space shards x%d + NCCL min-loc" % world,
            "l2": "flushed (256 MiB write) between timed steps"}


def free_port() -> int:
    import socket
    with socket.socket(socket.AF_INET, socket.SOCK_STREAM) as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


def relaunch_if_needed(args) -> None:
    """`python bench.py --gpus N` outside torchrun: re-exec under torch.distributed.run with N ranks
    (one GPU per rank), so the flag always means N processes."""
    if args.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=%d" % args.gpus,
           "--master-addr=127.0.0.1", "--master-port=%d" % free_port(), os.path.abspath(__file__)] + sys.argv[1:]
    sys.stdout.flush()
    os.execv(sys.executable, cmd)


def int_peak(local: int):
    """Measured integer peak (tools/int_peak.py): live on this GPU, plus the committed capture."""
    live = None
    try:
        from tools.int_peak import measure
        live = measure(local, target_ms=60.0)
    except Exception as exc:  # the product path does not depend on it; say why it is missing
        live = {"error": repr(exc)}
    saved = None
    try:
        with open(INT_PEAK_PATH) as fh:
            saved = json.load(fh)
    except (OSError, ValueError):
        pass
    return live, saved


def alu_peaks(live, saved):
    """(issue-bound int ops/s, ALU-pipe int ops/s, source) from the live run, else the committed one."""
    for src, d in (("measured live (tools/int_peak.py)", live), ("measured, profiles/int_peak.json", saved)):
        if d and "variants" in d:
            v = d["variants"]
            return (max(x["ops_per_s"] for x in v.values()),
                    next(x["ops_per_s"] for k, x in v.items() if k.startswith("alu (")), src)
    return None, None, "unavailable"


# ------------------------------------------------------------------------------------------------
# our arm
# ------------------------------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--state", default="a-nvlink", choices=["a-nvlink", "a-100g", "b"])
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-sample", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip the C1/C2/C3/C5 secondary measurements")
    ap.add_argument("--secondary", default="b", help="extra state measured in the same run ('' = none)")
    ap.add_argument("--dry-run", action="store_true", help="start the ranks and the process group, then exit")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    relaunch_if_needed(args)
    rank, world, local = env_int("RANK", 0), env_int("WORLD_SIZE", 1), env_int("LOCAL_RANK", 0)
    if world != args.gpus and not (args.gpus == 1 and "WORLD_SIZE" in os.environ):
        sys.stderr.write("bench.py: --gpus %d but WORLD_SIZE %d\n" % (args.gpus, world))
        sys.exit(2)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import numpy as np
    import torch
    import torch.distributed as dist

    import __graft_entry__
    __graft_entry__.build()
    import workloads as W
    from paper_conf_icpp_hulww24_b200 import Engine

    # AUTOPIPE_BENCH_BACKEND=gloo (test only): ranks may share a GPU (rank -> cuda:rank % count) so the
    # multi-rank path (shards, min-loc, max-over-ranks timing, one JSON line) runs on a 1-GPU box.
    # Its numbers are not scaling numbers; the driver's runs use NCCL, one GPU per rank.
    backend = os.environ.get("AUTOPIPE_BENCH_BACKEND", "nccl")
    if backend == "gloo":
        local = local % max(torch.cuda.device_count(), 1)
    if torch.cuda.is_available():
        torch.cuda.set_device(local)
    elif not (args.dry_run and backend == "gloo"):
        raise RuntimeError("bench.py needs a CUDA device (no CPU fallback)")
    dev = torch.device("cuda", local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if backend == "gloo":
            dist.init_process_group("gloo")
        else:
            os.environ.setdefault("NCCL_DEBUG", "INFO")  # the init log lets a reader count the ranks
            dist.init_process_group("nccl", device_id=dev)
        assert dist.get_world_size() == world
    if args.dry_run:  # launch check only: the ranks came up with one process group of the right size
        if rank == 0:
            print(json.dumps({"dry_run": True, "n_gpus": world, "backend": backend}), flush=True)
        if world > 1:
            dist.destroy_process_group()
        return
    from paper_conf_icpp_hulww24_b200.distributed import balanced_bounds

    from paper_conf_icpp_hulww24_b200 import result_from_bytes
    from paper_conf_icpp_hulww24_b200.distributed import minloc_device

    def barrier():
        if world > 1:
            if backend == "gloo":
                dist.barrier()
            else:
                dist.barrier(device_ids=[local])

    def max_over_ranks(x: float) -> float:
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.int32, device=dev)

    def measure_state(kind: str):
        prof, st = W.gpt96(), W.gpt_state(kind)
        eng = Engine(local)
        eng.load_profile(prof.O, prof.G, prof.P)
        # contiguous shards of about equal device cost under the state's integer path (the host
        # classifies it from the state; host-only estimate, any split gives the same optimum)
        eng.set_state(st.f, st.b, st.tau)
        bounds = balanced_bounds(96, 8, S_STAGES, S_STAGES, 0, world, eng.int_path)
        lo, hi = bounds[rank], bounds[rank + 1]
        d_fp = torch.tensor(np.asarray(st.f, dtype=np.uint64).view(np.int64), device=dev)
        d_bp = torch.tensor(np.asarray(st.b, dtype=np.uint64).view(np.int64), device=dev)
        d_tau = torch.tensor(np.asarray(st.tau, dtype=np.uint64).view(np.int64), device=dev)
        eng.set_timing(True)
        stream = torch.cuda.current_stream(dev)

        def step():
            # a1-a8 + e, all enqueued on the stream with no host wait: state kernel, the shard's
            # asynchronous search (result stays in device memory), and for N > 1 the device min-loc
            # (one NCCL all-gather of 40 B per rank + one reduction kernel)
            eng.set_state_device(d_fp, d_bp, d_tau)
            r = eng.search_optimum_async(S_STAGES, S_STAGES, 0, lo, hi)
            return minloc_device(r) if world > 1 else r

        for _ in range(args.warmup):
            step()
        torch.cuda.synchronize()
        barrier()
        eng.search_times()                         # drain the warm-up searches' kernel times
        launches0 = eng.kernel_launches
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        outs = []
        with ClockSampler(local) as clk:
            for k in range(args.steps):
                flush.fill_(k)                     # L2 flush: enqueued before the step's start event
                ev[k][0].record(stream)
                outs.append(step())
                ev[k][1].record(stream)
            torch.cuda.synchronize()
        barrier()
        # this library's kernels in the timed region: the context's (state, both gated search paths,
        # finalize) + the context-less min-loc reduction (one per step when N > 1)
        launches = eng.kernel_launches - launches0 + (args.steps if world > 1 else 0)
        kern_ms = eng.search_times()               # the K searches' enumeration kernels (CUDA events)
        assert len(kern_ms) == args.steps
        step_ms = [a.elapsed_time(b) for a, b in ev]
        rank_total_ms = sum(step_ms)
        total_ms = max_over_ranks(rank_total_ms)
        kern_avg = max_over_ranks(sum(kern_ms) / len(kern_ms))
        results = [(r.time_ns, r.index) for r in map(result_from_bytes, outs)]
        assert all(x == results[0] for x in results), "non-deterministic optimum"
        assert all(result_from_bytes(o).evaluated == (TOTAL if world > 1 else hi - lo) for o in outs)
        # e2e: the public API from host buffers (profile + state copied every step, the 40-byte
        # result read back to the host)
        # the step's inputs as a user holds them: uint64 host arrays (Table 1 rows), copied to the
        # device by the calls inside the timed region (staged through the context's pinned buffers)
        h_O, h_G, h_P = (np.asarray(x, dtype=np.uint64) for x in (prof.O, prof.G, prof.P))
        h_f, h_b, h_tau = (np.asarray(x, dtype=np.uint64) for x in (st.f, st.b, st.tau))
        t_e2e = []
        for k in range(args.steps):
            flush.fill_(k)
            torch.cuda.synchronize()
            barrier()
            t0 = time.perf_counter()
            eng.load_profile(h_O, h_G, h_P)
            eng.set_state(h_f, h_b, h_tau)
            r = eng.search_optimum_async(S_STAGES, S_STAGES, 0, lo, hi)
            best = result_from_bytes(minloc_device(r) if world > 1 else r)
            t_e2e.append(time.perf_counter() - t0)
            assert (best.time_ns, best.index) == results[0]
        e2e_s = max_over_ranks(sum(t_e2e))
        int_path = eng.int_path
        eng.close()
        h2d = 3 * 96 * 8 + 2 * 8 * 96 * 8 + 8 * 8 * 8
        return {"total_ms": total_ms, "ms_per_step": total_ms / args.steps, "kernel_ms": kern_avg, "cands": hi - lo,
                "value": TOTAL * args.steps / (total_ms / 1000.0), "optimum": results[0],
                "launches": launches, "clocks": clk.summary(), "int_path": int_path,
                "e2e": {"value": TOTAL * args.steps / e2e_s, "unit": UNIT, "h2d_bytes_per_step": h2d,
                        "d2h_bytes_per_step": 40, "ms_per_step": 1000 * e2e_s / args.steps}}

    main_res = measure_state(args.state)
    extra = {}
    if args.secondary and args.secondary != args.state:
        s2 = measure_state(args.secondary)
        extra[args.secondary] = {"value": s2["value"], "ms_per_step": s2["ms_per_step"],
                                 "int_path": s2["int_path"], "optimum_T_ns": s2["optimum"][0],
                                 "optimum_index": s2["optimum"][1], "kernel_ms": s2["kernel_ms"],
                                 "e2e_value": s2["e2e"]["value"], "clocks": s2["clocks"]}

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return

    # roofline of the dominant kernel (k_search_r1), against the measured integer peak
    live, saved = int_peak(local)
    peaks = {}
    try:
        with open(PEAKS_PATH) as fh:
            peaks = json.load(fh)
    except (OSError, ValueError):
        pass
    peak_issue, peak_alu, peak_src = alu_peaks(live, saved)
    ops_per_cand = OPS_PER_CANDIDATE[main_res["int_path"]]
    cands_per_rank = main_res["cands"]
    achieved = ops_per_cand * cands_per_rank / (main_res["kernel_ms"] / 1000.0) / 1e12
    kname = "k_search_r1<8,%s>" % ("u32" if main_res["int_path"] == 32 else "u64")
    traffic = None
    try:
        with open(TRAFFIC_PATH) as fh:
            traffic = json.load(fh).get(kname)
    except (OSError, ValueError):
        pass
    peak_t = peak_issue / 1e12 if peak_issue else None
    frac = achieved / peak_t if peak_t else None
    ncu = ncu_kernel_metrics(("k_search_r1<8, unsigned int" if main_res["int_path"] == 32
                              else "k_search_r1<8, unsigned long long"))
    roofline = {"bound": "alu", "achieved": achieved, "peak": peak_t, "unit": "Tops/s", "frac": frac,
                "traffic": traffic, "traffic_unit": "bytes per launch (ncu dram read + write)",
                "kernel": kname, "ops_per_candidate": ops_per_cand,
                "ops_unit": "SURVEY.md §8(d): incremental full-T evaluation of one S = 8, r = 1 candidate "
                            "(85 int ops on the 32-bit path, 170 on the 64-bit one)",
                "decision_only": True,
                "frac_exceeds_1": bool(frac and frac > 1.0),
                "note": "the kernel decides T <= theta per candidate without computing T (exact T only on "
                        "the rare path), so it does less than the algorithmic unit per candidate and the "
                        "fraction is not bounded by 1; its issue-slot use is in profiles/round2_kernels_full.txt",
                "peak_source": peak_src, "peak_alu_pipe_only": peak_alu / 1e12 if peak_alu else None,
                "kernel_ms": main_res["kernel_ms"], "candidates_per_launch": cands_per_rank,
                "ncu": ncu}

    configs = None
    if world == 1 and not args.no_configs:
        from tools.bench_configs import measure as measure_configs
        configs = measure_configs(local)
        for v in configs.values():
            v.pop("per_state", None)
        # full-T roofline of the bulk-scoring kernel (k_eval on the C5 rollout batch): every record's
        # T is computed; ALU at 230 int ops per record and HBM at 24 B per record
        c5 = configs.get("C5_resnet50_rollout")
        if c5:
            rps = c5["eval_records_per_s"]
            ops = rps * ROLLOUT_OPS / 1e12
            gbs = rps * ROLLOUT_BYTES / 1e9
            hbm = float(peaks.get("hbm_gbs", 0)) or None
            c5["roofline"] = {"bound": "alu", "kernel": "k_eval<PipeDream,u64>", "achieved": ops, "unit": "Tops/s",
                              "peak": peak_t, "frac": ops / peak_t if peak_t else None,
                              "ops_per_record": ROLLOUT_OPS, "bytes_per_record": ROLLOUT_BYTES,
                              "achieved_GBps": gbs, "hbm_peak_GBps": hbm,
                              "hbm_frac": gbs / hbm if hbm else None, "peak_source": peak_src,
                              "decision_only": False}
        # the same roofline on the records the 230-op unit describes (S = 8, r = 1, GPT-96, u32 path)
        c4 = configs.get("C4_gpt96_r1_records")
        if c4:
            rps = c4["eval_records_per_s"]
            ops = rps * ROLLOUT_OPS / 1e12
            gbs = rps * ROLLOUT_BYTES / 1e9
            hbm = float(peaks.get("hbm_gbs", 0)) or None
            c4["roofline"] = {"bound": "alu", "kernel": "k_eval<PipeDream,u32>", "achieved": ops, "unit": "Tops/s",
                              "peak": peak_t, "frac": ops / peak_t if peak_t else None,
                              "ops_per_record": ROLLOUT_OPS, "bytes_per_record": ROLLOUT_BYTES,
                              "achieved_GBps": gbs, "hbm_peak_GBps": hbm,
                              "hbm_frac": gbs / hbm if hbm else None, "peak_source": peak_src,
                              "decision_only": False,
                              "note": "every record is an S = 8, r = 1 partition: the unit's own case"}

    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        v, n, dt, nc = oracle_throughput(args.state)
        dp_s, dpT, dpI = param_dp_time(args.state)
        assert (dpT, dpI) == tuple(main_res["optimum"]), "GPU optimum differs from the oracle's parametric DP"
        cpu = {"value": v, "unit": UNIT, "cores": nc, "kind": "oracle",
               "sample": "%d seeded random candidates of the C(95,7) space, event simulation, %.1f s" % (n, dt),
               "cpu": cpu_model(),
               "extrapolated_exhaustive_s": TOTAL / v,
               "param_dp_time_to_optimum_s_1core": dp_s}

    line = {
        "metric": METRIC, "value": main_res["value"], "unit": UNIT, "n_gpus": world,
        "decision_only": True, "decided_per_s": main_res["value"],
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": main_res["ms_per_step"],
        "time_to_optimum_ms": main_res["ms_per_step"],
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "u32" if main_res["int_path"] == 32 else "u64", "data": "synthetic",
        "config": config_block(args, world),
        "optimum": {"T_ns": main_res["optimum"][0], "index": main_res["optimum"][1]},
        "gpu_launches": main_res["launches"],
        "clocks": main_res["clocks"],
        "e2e": main_res["e2e"],
        "roofline": roofline,
        "cpu_baseline": cpu,
        "int_peak": {"live": live, "committed": saved and {k: saved.get(k) for k in
                                                            ("peak_int_ops_per_s", "alu_pipe_ops_per_s", "clocks")}},
        "secondary_states": extra,
        "configs": configs,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
