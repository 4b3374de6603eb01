"""bench.py's launch contract (task statement): `--gpus N` outside torchrun
re-executes under torch.distributed.run with N ranks, so the flag always means N processes. The CPU
test brings the ranks and a gloo process group up (--dry-run); the GPU test runs the whole bench step
with 2 ranks sharing the box's GPU (gloo) and checks the optimum equals the 1-rank run's."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, timeout=600):
    env = dict(os.environ, AUTOPIPE_BENCH_BACKEND="gloo")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                       timeout=timeout, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_gpus_flag_launches_ranks():
    assert _run(["--gpus", "2", "--dry-run"], timeout=300)["n_gpus"] == 2


@pytest.mark.gpu
def test_gpus_flag_same_optimum():
    common = ["--steps", "3", "--warmup", "3", "--no-configs", "--no-cpu-baseline", "--secondary", ""]
    one = _run(["--gpus", "1"] + common)
    two = _run(["--gpus", "2"] + common)
    assert one["n_gpus"] == 1 and two["n_gpus"] == 2
    assert one["optimum"] == two["optimum"]
