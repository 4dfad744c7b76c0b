"""GPU parity of both GEMM1 schedules: single row-blocks and pairs of row-blocks sharing each K tile
(`SR_G1_PAIR`, read once per process, so each mode runs in its own interpreter).  The library picks
pairs by default only for D = 128; here every case runs in both modes whatever its D."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import workloads as W
from tests.test_gpu_parity import run_case, assert_close
cases = [
    ("dense", 1, 2, 640, 128, "bf16", dict(causal=True)),                 # odd row-block count
    ("dense", 2, 1, 512, 64, "f16", dict(kv_len=[300, 1])),
    ("dense", 1, 2, 384, 128, "f16", dict(tile_n=64, causal=True)),
    ("window", 1, 2, 1024, 64, "f16", dict(window=128, n_global=8)),
    ("window", 1, 1, 768, 64, "f16", dict(window=126, n_global=8, tile_n=64, fused=False)),
    ("block", 1, 2, 768, 64, "f16", dict(layout=W.random_layout(2, 768 // 64, 64, 0.3, seed=5))),
    # the paper's standalone IR kernel (SR_IR_KERNEL) on each schedule
    ("dense", 1, 2, 640, 128, "bf16", dict(causal=True, ir_kernel=True)),
    ("dense", 2, 1, 512, 64, "f16", dict(kv_len=[300, 1], ir_kernel=True)),
    ("dense", 1, 2, 384, 128, "f16", dict(tile_n=64, causal=True, ir_kernel=True)),
    ("block", 1, 2, 768, 64, "f16", dict(layout=W.random_layout(2, 768 // 64, 64, 0.3, seed=5), ir_kernel=True)),
]
for kind, B, H, S, D, dt, kw in cases:
    o, ref = run_case(kind, B, H, S, D, dt, **kw)
    assert_close(o, ref, dt, what=f"{kind} {kw}")
print("ok", len(cases))
"""


@pytest.mark.parametrize("mode", ["0", "1"], ids=["single", "pairs"])
def test_gemm1_schedules(mode):
    env = dict(os.environ, SR_G1_PAIR=mode, PYTHONPATH=ROOT)
    r = subprocess.run([sys.executable, "-c", SCRIPT], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=240)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]
