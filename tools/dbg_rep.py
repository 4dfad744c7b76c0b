"""Repeat one config's recomposed layer N times and count runs whose sampled rows exceed 1e-2."""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import oracle, workloads as W  # noqa
from tests.test_gpu_parity import _config_call, _sample_rows  # noqa
idx, n = int(sys.argv[1]), int(sys.argv[2])
cfg = W.config(idx); t = W.config_tensors(cfg)
rows = _sample_rows(cfg, 2048, seed=5)
o, m = _config_call(cfg, t, fused=True)
ref = oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, m)
ridx = torch.from_numpy(rows).cuda()
nbad = 0
for r in range(n):
    o, _ = _config_call(cfg, t, fused=True)
    got = o.reshape(-1, cfg.D)[ridx].double().cpu().numpy()
    err = np.abs(got - ref).max(axis=1)
    bad = rows[err > 1e-2]
    if len(bad):
        nbad += 1
        print("run", r, "bad", [(int(x // cfg.S), int(x % cfg.S)) for x in bad[:6]], "max", err.max())
print(f"C{idx}: {nbad}/{n} runs with bad rows")
