import sys
import torch
sys.path.insert(0, '.')
import workloads as W, paper_conf_iiswc_choilkha22_b200 as sr  # noqa
from tests.gpu_util import to_dev  # noqa
idx, n, T = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
cfg = W.config(idx); t = W.config_tensors(cfg)
mask = (sr.window_mask(cfg.window, cfg.n_global) if cfg.kind == "window" else
        sr.block_mask(W.config_layout(cfg)) if cfg.kind == "blocksparse" else sr.dense_mask(cfg.kv_len))
dt = {"f16": sr.SR_F16, "bf16": sr.SR_BF16}[cfg.dtype]
info = sr.workspace_info(mask, cfg.B, cfg.H, cfg.S, cfg.D, dt, causal=cfg.causal, tile_n=T)
ws = torch.zeros(info["total_bytes"], dtype=torch.uint8, device="cuda")
q0, k0, v0 = (to_dev(x, cfg.dtype) for x in (t.q_s, t.k_s, t.v_s))
run = lambda st: sr.call(mask, q0, k0, v0, scale=cfg.scale, causal=cfg.causal, workspace=ws, stages=st, tile_n=T)
run(0); torch.cuda.synchronize()
base = run(4).clone()
tot = 0
for k in range(n):
    o = run(4); torch.cuda.synchronize()
    rows = torch.nonzero((o != base).reshape(-1, cfg.D).any(dim=1)).flatten().cpu().tolist()
    tot += bool(rows)
print(f"C{idx} T={T}: differing runs {tot} of {n}")
