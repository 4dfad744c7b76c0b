"""Print max |gpu - oracle| of the training backward per case (diagnostic companion of
tests/test_gpu_backward.py):  python tools/bwd_errors.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import workloads as W  # noqa: E402
from tests.test_gpu_backward import run_bwd  # noqa: E402

cases = [("dense causal kv f16 D64", dict(kind="dense", B=2, H=2, S=384, D=64, dtype="f16", causal=True, kv_len=[384, 200])),
         ("dense causal bf16 D128", dict(kind="dense", B=2, H=2, S=384, D=128, dtype="bf16", causal=True)),
         ("dense T64 f16", dict(kind="dense", B=1, H=3, S=512, D=64, dtype="f16", kv_len=[449], tile_n=64)),
         ("block f16", dict(kind="block", B=1, H=2, S=512, D=64, dtype="f16", layout=W.random_layout(2, 8, 64, 0.35, seed=5))),
         ("window f16", dict(kind="window", B=1, H=2, S=640, D=64, dtype="f16", window=128, n_global=8))]
for name, c in cases:
    kind = c.pop("kind")
    B, H, S, D, dt = (c.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    got, ref = run_bwd(kind, B, H, S, D, dt, **c)
    print(name, {n: (f"{np.abs(g - r).max():.3g}", f"{np.abs(r).max():.3g}") for n, g, r in zip(("O", "dQ", "dK", "dV"), got, ref)})
