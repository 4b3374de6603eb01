"""CPU (`-m "not gpu"`) checks of the GPU path's round-robin recurrence (rr.cuh, row f4, reading F-5):
the header compiled for the host with g++ (tests/host: a shim for the CUDA qualifiers and intrinsics)
scores seeded C5 records of four rollout states and random small instances, and every T must equal
the oracle's (oracle/roundrobin.py). Run plain and with UBSan/ASan, and with a 3-round budget so
every replicated record goes through the growth-bound bracket and the Bellman-Ford search (the path
of the GPU's deferred and long-transient records). The host build cannot see device-compiler
behaviour (an NVVM -O3 miscompile of an earlier version passed here); the GPU parity
tests remain the gate."""
import os
import shutil
import subprocess

import numpy as np
import pytest

import workloads as W
from tests._oracle_pool import rr_many

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(ROOT, "paper_conf_icpp_hulww24_b200", "csrc")

pytestmark = pytest.mark.skipif(shutil.which("g++") is None, reason="needs g++")


def _build(tmp, flags, name):
    exe = os.path.join(tmp, name)
    cmd = ["g++", "-std=c++17", "-w", "-I" + os.path.join(HERE, "host", "inc"), "-I" + CSRC, "-include",
           os.path.join(HERE, "host", "cuda_host_shim.h"), os.path.join(HERE, "host", "rr_host.cpp"), "-o", exe] + flags
    subprocess.run(cmd, check=True, capture_output=True, text=True)
    return exe


def _dump(path, prof, st, recs, sync=0):
    ref = rr_many(prof, st, recs, sync)
    with open(path, "w") as f:
        f.write("%d %d\n" % (len(prof.O), len(st.f)))
        for rows in (st.f, st.b):
            f.write(" ".join(str(x) for row in rows for x in row) + "\n")
        for arr in (prof.O, prof.G, prof.P):
            f.write(" ".join(map(str, arr)) + "\n")
        f.write(" ".join(str(x) for row in st.tau for x in row) + "\n")
        f.write("%d %d\n" % (len(recs), sync))
        for r, t in zip(recs, ref):
            f.write("%x %x %d\n" % (int.from_bytes(r[:8], "little"), int.from_bytes(r[8:], "little"), t))


@pytest.fixture(scope="module")
def dumps(tmp_path_factory):
    tmp = str(tmp_path_factory.mktemp("rr_host"))
    paths = []
    prof = W.resnet50()
    for k in range(4):  # C5 rollout states, seeded records (+ the long-transient record on state 0)
        st = W.rollout_state(prof, k)
        recs = [bytes(r) for r in W.sample_records(prof.L, st.N, 250, 3000 + k)]
        if k == 0:
            recs.append(W.encode(3, [15, 29], [1, W.IDLE, 2, 1, 0]))
        paths.append(os.path.join(tmp, "c5_%d.txt" % k))
        _dump(paths[-1], prof, st, recs)
    rng = np.random.default_rng(4100)
    for k in range(3):  # random small instances, both sync schemes
        L, N = int(rng.integers(3, 12)), int(rng.integers(2, 9))
        prof = W.random_profile(L, rng, f_max=int(rng.choice([300, 10**6])), bytes_max=int(rng.choice([10**3, 10**7])))
        st = W.random_state_small(prof, N, rng, tau_max=int(rng.choice([200, 10**5])))
        recs = [bytes(r) for r in W.sample_records(L, N, 200, int(rng.integers(1 << 30)))]
        paths.append(os.path.join(tmp, "rnd_%d.txt" % k))
        _dump(paths[-1], prof, st, recs, sync=k % 2)
    return tmp, paths


@pytest.mark.parametrize("mode", ["O2", "sanitized", "budget3"])
def test_host_rr_matches_oracle(dumps, mode):
    tmp, paths = dumps
    flags = {"O2": ["-O2"], "sanitized": ["-O1", "-g", "-fsanitize=undefined,address", "-fno-sanitize-recover=all"],
             "budget3": ["-O2"]}[mode]
    exe = _build(tmp, flags, "rr_" + mode)
    for path in paths:
        args = [exe, path] + (["3"] if mode == "budget3" else [])
        r = subprocess.run(args, capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, (path, r.stdout[-2000:], r.stderr[-2000:])
        assert "bad 0" in r.stdout
