import sys
import torch
sys.path.insert(0, '.')
import workloads as W, paper_conf_iiswc_choilkha22_b200 as sr  # noqa
from tests.gpu_util import to_dev  # noqa
idx, n = int(sys.argv[1]), int(sys.argv[2])
cfg = W.config(idx); t = W.config_tensors(cfg)
mask = sr.window_mask(cfg.window, cfg.n_global) if cfg.kind == "window" else sr.block_mask(W.config_layout(cfg))
info = sr.workspace_info(mask, cfg.B, cfg.H, cfg.S, cfg.D, sr.SR_F16)
ws = torch.zeros(info["total_bytes"], dtype=torch.uint8, device="cuda")
q0, k0, v0 = (to_dev(x, cfg.dtype) for x in (t.q_s, t.k_s, t.v_s))
run = lambda st: sr.call(mask, q0, k0, v0, scale=cfg.scale, workspace=ws, stages=st)
run(0); torch.cuda.synchronize()
base = run(4).clone()
tot = 0
for k in range(n):
    o = run(4); torch.cuda.synchronize()
    rows = torch.nonzero((o != base).reshape(-1, cfg.D).any(dim=1)).flatten().cpu().tolist()
    if rows:
        tot += 1
        g = sorted(set((r // cfg.S, (r % cfg.S) // 128) for r in rows))
        print("run", k, len(rows), "rows; (head,rowblock):", g[:4], "lanes:", sorted(set(r % 128 for r in rows))[:40], flush=True)
print("differing runs", tot, "of", n)
