#!/usr/bin/env python
"""Measured integer-ALU peak of the GPU: runs tools/int_peak.cu's
independent-chain kernels on every SM at full occupancy, logs SM clocks during each run, reads the
per-trip op count from the source and the SASS total, and writes profiles/int_peak.json.

  python tools/int_peak.py [--out profiles/int_peak.json]

bench.py calls measure() live (a few hundred ms) for the denominator of its ALU rooflines.
"""
from __future__ import annotations

import argparse
import collections
import ctypes
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "tools", "int_peak.cu")
LIB = os.path.join(ROOT, "tools", "libintpeak.so")
VARIANTS = {0: "alu (IADD/VIADD, LOP3, VIMNMX)", 1: "alu+fma (the above 1:1 with IMAD)", 2: "isetp (VIADD, ISETP, SEL)"}
KERNELS = {0: "k_int_alu", 1: "k_int_mix", 2: "k_int_cmp"}


def build() -> str:
    if not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
        subprocess.run([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-Xcompiler", "-fPIC",
                        "-shared", "-o", LIB, SRC], check=True, capture_output=True)
    return LIB


def sass_ops_per_trip() -> dict:
    """Integer instructions in each kernel's loop body, counted from the SASS (the unrolled body is
    the only block with more than 90 ALU/FMA instructions)."""
    try:
        txt = subprocess.run(["cuobjdump", "-sass", build()], capture_output=True, text=True, check=True).stdout
    except (OSError, subprocess.CalledProcessError):
        return {}
    out, cur = {}, None
    count = collections.Counter()
    pat = re.compile(r"/\*[0-9a-f]{4}\*/\s+(?:@!?U?P\w+\s+)?([A-Z0-9_]+)")
    for line in txt.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = m.group(1)
            continue
        m = pat.search(line)
        if m and cur:
            count[(cur, m.group(1))] += 1
    for v, k in KERNELS.items():
        ops = sum(n for (f, op), n in count.items() if k in f and op in
                  ("VIADD", "IADD3", "LOP3", "VIMNMX", "IMAD", "ISETP", "SEL"))
        out[v] = ops
    return out


def measure(device: int = 0, target_ms: float = 150.0, sampler=None) -> dict:
    """Runs the three variants; returns {variant: {...ops_per_s...}} plus the clocks seen."""
    import torch
    lib = ctypes.CDLL(build())
    lib.int_peak_run.restype = ctypes.c_float
    lib.int_peak_run.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int]
    lib.int_peak_ops_per_trip.restype = ctypes.c_int
    torch.cuda.set_device(device)
    props = torch.cuda.get_device_properties(device)
    sms = props.multi_processor_count
    blocks = sms * 8  # 2048 resident threads per SM
    sass = sass_ops_per_trip()
    res = {"sms": sms, "blocks": blocks, "threads_per_block": 256, "gpu": props.name, "variants": {}}
    for v in VARIANTS:
        ops_trip = lib.int_peak_ops_per_trip(v)
        ms = lib.int_peak_run(v, blocks, 64)
        iters = max(64, int(64 * target_ms / max(ms, 1e-3)))
        ms = lib.int_peak_run(v, blocks, iters)
        if ms <= 0:
            raise RuntimeError("int_peak_run failed")
        ops = blocks * 256 * iters * ops_trip
        res["variants"][VARIANTS[v]] = {"ops_per_thread_trip": ops_trip, "sass_int_ops_in_kernel": sass.get(v),
                                        "iters": iters, "ms": ms, "ops_per_s": ops / (ms / 1e3)}
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "int_peak.json"))
    ap.add_argument("--device", type=int, default=0)
    args = ap.parse_args()
    sys.path.insert(0, ROOT)
    from bench import ClockSampler
    with ClockSampler(args.device, 0.01) as clk:
        res = measure(args.device, target_ms=400.0)
    res["clocks"] = clk.summary()
    mhz = res["clocks"].get("sm_mhz") or 1965.0
    for v in res["variants"].values():
        v["lanes_per_sm_per_clk"] = v["ops_per_s"] / (res["sms"] * mhz * 1e6)
    res["peak_int_ops_per_s"] = max(v["ops_per_s"] for v in res["variants"].values())
    res["alu_pipe_ops_per_s"] = res["variants"][VARIANTS[0]]["ops_per_s"]
    res["how"] = ("tools/int_peak.cu: 8 independent dependency chains per thread, 2048 threads per SM on every "
                  "SM, ops per loop trip from the source (checked against the SASS count), CUDA events; "
                  "peak_int_ops_per_s = best variant (ALU + FMA pipes = the issue bound), "
                  "alu_pipe_ops_per_s = the ALU pipe alone")
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as fh:
        json.dump(res, fh, indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
