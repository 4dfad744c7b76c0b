"""Debug aid: run one config's recomposed layer and compare m', d', r' and O of selected heads with
the oracle's Eq. (2) decomposition.  python tools/debug_intermediates.py CFG [heads]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Layer, oracle_mask_for  # noqa: E402

idx = int(sys.argv[1])
nh = int(sys.argv[2]) if len(sys.argv) > 2 else 1
cfg = W.config(idx)
L = Layer(cfg, torch.device("cuda", 0), cfg.idx, sr, torch)
o = torch.empty(cfg.B, cfg.H, cfg.S, cfg.D, dtype=torch.float32, device="cuda")
sr.call(L.mask, L.dev["q"], L.dev["k"], L.dev["v"], out=o, out_dtype=torch.float32, workspace=L.ws[True], **L.kw)
torch.cuda.synchronize()
tdt = {"f16": torch.float16, "bf16": torch.bfloat16, "f32": torch.float32}[cfg.dtype]
info = sr.workspace_info(L.mask, cfg.B, cfg.H, cfg.S, cfg.D, sr.dtype_code(tdt), causal=cfg.causal)
T = info["tile_n"]
ws = L.ws[True]
n = info["n_slots"] * 128
get = lambda key: ws[info[key]:].view(torch.float32)[:n].cpu().numpy().reshape(cfg.BH, -1, 128)
mp, dp, rp = get("off_mprime"), get("off_dprime"), get("off_rprime")
t = W.config_tensors(cfg)
sub = lambda x: x.reshape(cfg.BH, cfg.S, cfg.D)[:nh].reshape(1, nh, cfg.S, cfg.D)
m = oracle_mask_for(cfg)
if cfg.kind == "blocksparse":
    lay = W.config_layout(cfg)
    m = oracle.Mask(kind="block", layout=W.csr_from_sets(64, [[lay.blocks(h, r) for r in range(lay.nb)] for h in range(nh)]))
ref, mr, dr, rr = oracle.recomposed(sub(t.q64), sub(t.k64), sub(t.v64), cfg.scale, T, m)
# schedule of the GPU: tiles per row-block from schedule lists (host mirror through tile counting)
og = o.reshape(cfg.BH, cfg.S, cfg.D)[:nh].cpu().numpy()
err = np.abs(og - ref.reshape(nh, cfg.S, cfg.D))
bad_rows = np.unique(np.nonzero(err > 1e-2)[1])
print("O max err", err.max(), "bad rows", bad_rows[:40], len(bad_rows))
# compare r' per (row, tile) using the oracle's kt index: GPU slot order = tile list order per row-block
a = oracle_np = None
from oracle import oracle_np as onp  # noqa: E402
for g in range(nh):
    allowed = onp.allowed_matrix(cfg.S, h=g, **({"kind": "window", "window": cfg.window, "n_global": cfg.n_global}
                                                  if cfg.kind == "window" else {"kv_len": cfg.kv_len, "causal": cfg.causal}
                                                  if cfg.kind == "dense" else {"kind": "block", "layout": lay}))
    slot = 0
    worst = (0, None)
    for rb in range(cfg.S // 128):
        for kt in range(cfg.S // T):
            blk = allowed[rb * 128:(rb + 1) * 128, kt * T:(kt + 1) * T]
            hv = [blk[:64].any(), blk[64:].any()]
            if not any(hv):
                continue
            rows = np.arange(rb * 128, rb * 128 + 128)
            for h in range(2):
                if not hv[h]:
                    continue
                rs = rows[h * 64:(h + 1) * 64]
                e_r = np.abs(rp[g, slot, h * 64:(h + 1) * 64] - rr[g, kt, rs])
                e_m = np.abs(np.where(np.isinf(mr[g, kt, rs]), 0, mp[g, slot, h * 64:(h + 1) * 64] - mr[g, kt, rs]))
                e_d = np.abs(dp[g, slot, h * 64:(h + 1) * 64] - dr[g, kt, rs]) / np.maximum(dr[g, kt, rs], 1e-30)
                w = max(e_r.max(), 0)
                if w > worst[0]:
                    worst = (w, (rb, kt, h, e_m.max(), e_d.max()))
            slot += 1
    print("head", g, "worst r' abs err", worst)
