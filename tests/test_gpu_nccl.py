"""Row e's NCCL code path on the one GPU a test box has: a process group of world size 1 over the
"nccl" backend runs `minloc_device` (all_gather_into_tensor of the 40-byte result, then the device
reduction autopipe_reduce_results), `bound_allreduce` (all_reduce MIN of the seed word) and
`rollout_distributed` (all_gather_into_tensor of the padded per-rank output slices) exactly as an
8-rank job does, minus the other ranks. The 96-layer 8-stage optimum (C4b, 64-bit path) must equal
the oracle's parametric DP, through both the plain and the bounded search. (Several ranks on one GPU
cannot share an NCCL communicator; the multi-rank exchange itself is covered by the gloo tests.)"""
import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu

SCRIPT = r"""
import json, sys
sys.path.insert(0, %(root)r)
import torch, torch.distributed as dist
import workloads as W
from paper_conf_icpp_hulww24_b200 import Engine
from paper_conf_icpp_hulww24_b200.distributed import (search_distributed, balanced_bounds, bound_allreduce,
                                                      minloc_device)
from paper_conf_icpp_hulww24_b200 import result_from_bytes
torch.cuda.set_device(0)
dist.init_process_group("nccl", init_method="tcp://127.0.0.1:%(port)d", rank=0, world_size=1,
                        device_id=torch.device("cuda", 0))
assert dist.get_backend() == "nccl"
eng = Engine(0)
prof, st = W.gpt96(), W.gpt_state("b")
eng.load(prof, st)
r = search_distributed(eng, 8, 8)
b = balanced_bounds(96, 8, 8, 8, 0, 1)
theta = bound_allreduce(eng.search_seed_async(8, 8, begin=b[0], end=b[1]))
eng.set_search_bound(theta)
rb = result_from_bytes(minloc_device(eng.search_optimum_async(8, 8, begin=b[0], end=b[1])))
eng.set_search_bound(None)
from paper_conf_icpp_hulww24_b200.distributed import rollout_distributed
rp = W.resnet50()
rst = W.rollout_state(rp, 0)
eng.load(rp, rst)
recs = torch.from_numpy(W.sample_records(rp.L, rst.N, 5000, 1000)).cuda()
rt, rsw = rollout_distributed(eng, recs, bytes(recs[0].cpu().numpy()))
torch.cuda.synchronize()
m = (1 << 64) - 1
print(json.dumps({"T": r.time_ns, "idx": r.index, "n": r.evaluated, "Tb": rb.time_ns, "idxb": rb.index,
                  "nb": rb.evaluated, "part": list(r.partition),
                  "rt": [int(x) & m for x in rt.cpu()], "rsw": [int(x) & m for x in rsw.cpu()]}))
dist.destroy_process_group()
"""


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_nccl_minloc_and_bound_world1():
    from oracle import param_dp
    import workloads as W
    from oracle.model import parse_record
    code = SCRIPT % {"root": ROOT, "port": _free_port()}
    p = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert p.returncode == 0, p.stderr[-3000:]
    got = json.loads([ln for ln in p.stdout.splitlines() if ln.startswith("{")][-1])
    prof, st = W.gpt96(), W.gpt_state("b")
    T, idx, part = param_dp.optimum(prof, st, 8, 8)
    assert (got["T"], got["idx"], got["n"]) == (T, idx, 11_050_084_695)
    assert (got["Tb"], got["idxb"], got["nb"]) == (T, idx, 11_050_084_695)
    assert parse_record(bytes(got["part"]), 96, 8) == part
    # rollout_distributed (row e for rollout batches) through NCCL: the gathered batch, sampled
    from tests._oracle_pool import rollout_many
    rp = W.resnet50()
    rst = W.rollout_state(rp, 0)
    recs = W.sample_records(rp.L, rst.N, 5000, 1000)
    idx = list(range(0, 5000, 7))
    ot, osw = rollout_many(rp, rst, [bytes(recs[i]) for i in idx], bytes(recs[0]))
    assert len(got["rt"]) == len(got["rsw"]) == 5000
    assert [got["rt"][i] for i in idx] == ot and [got["rsw"][i] for i in idx] == osw
