"""bench.py's N > 1 path (head-sharded layer, max over ranks, weak-scaling field) under torchrun with
two ranks.  On a one-GPU box both ranks share cuda:0 (SR_BENCH_SHARED_GPU=1, gloo for the host-side
plumbing): a functional check of the sharding and reporting code, not a timing."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("config", [2, 4])
def test_bench_two_ranks(config):
    env = dict(os.environ, SR_BENCH_SHARED_GPU="1", PYTHONPATH=ROOT)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(29600 + config), "bench.py", "--gpus", "2",
           "--steps", "3", "--warmup", "3", "--config", str(config)]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["value"] > 0
    assert d["config"]["parallelism"].startswith("heads2")
    assert d["weak"]["value"] > 0
    assert d["gpu_launches"] > 0
