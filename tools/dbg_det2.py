import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import workloads as W  # noqa
from tests.test_gpu_parity import _config_call  # noqa
idx, n = int(sys.argv[1]), int(sys.argv[2])
cfg = W.config(idx); t = W.config_tensors(cfg)
for od in (True, False):
    o0 = None
    for k in range(n):
        o, _ = _config_call(cfg, t, fused=True, out_f32=od)
        o = o.float()
        if o0 is None:
            o0 = o.clone(); continue
        d = (o != o0)
        rows = torch.nonzero(d.reshape(-1, cfg.D).any(dim=1)).flatten().cpu().numpy()
        print("f32out" if od else "dtypeout", "run", k, "rows differing:", len(rows), [(int(r // cfg.S), int(r % cfg.S)) for r in rows[:5]],
              "max diff", float((o - o0).abs().max()), flush=True)
