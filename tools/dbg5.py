import sys, numpy as np, torch
sys.path.insert(0, '.')
import oracle, workloads as W, paper_conf_iiswc_choilkha22_b200 as sr
from tests.test_gpu_parity import _config_call, _sample_rows
for order in ([5], [4, 5]):
    for idx in order:
        cfg = W.config(idx); t = W.config_tensors(cfg)
        o, m = _config_call(cfg, t, fused=True)
    rows = _sample_rows(cfg, 192, seed=5)
    ref = oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, m)
    got = o.reshape(-1, cfg.D)[torch.from_numpy(rows).cuda()].double().cpu().numpy()
    err = np.abs(got - ref).max(axis=1)
    bad = rows[err > 1e-2]
    print(order, "bad rows (g, i):", [(int(r // cfg.S), int(r % cfg.S)) for r in bad], "max", err.max())
