"""A/B timing of library builds on one box (SR_MHA_LIB selects the .so; run one process per build):
    SR_MHA_LIB=path python tools/ab_time.py CFG [K] [modes]
Back-to-back layers (one CUDA graph of K calls cycling through input/workspace sets larger than 2x
L2), median of 5 regions; modes: default, two_kernels, ir_kernel, unfused (comma list)."""
import math
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402

idx = int(sys.argv[1])
K = int(sys.argv[2]) if len(sys.argv) > 2 else 20
modes = (sys.argv[3] if len(sys.argv) > 3 else "default,two_kernels,ir_kernel,unfused").split(",")
cfg = W.config(idx)
dev = torch.device("cuda", 0)
tdt = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}[cfg.dtype]
mask = (sr.dense_mask(cfg.kv_len) if cfg.kind == "dense" else sr.block_mask(W.config_layout(cfg))
        if cfg.kind == "blocksparse" else sr.window_mask(cfg.window, cfg.n_global))
KW = {"default": dict(), "two_kernels": dict(two_kernels=True, tile_n=64 if cfg.kind == "blocksparse" else 128),
      "ir_kernel": dict(ir_kernel=True, tile_n=64 if cfg.kind == "blocksparse" else 128),
      "unfused": dict(fused=False, tile_n=64)}


def tens(seed):
    t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=seed)
    out = []
    for a in (t.q_s, t.k_s, t.v_s):
        x = torch.from_numpy(a.view(np.int16).copy()).view(torch.bfloat16) if cfg.dtype == "bf16" else torch.from_numpy(a)
        out.append(x.to(dev))
    return out


base = tens(cfg.idx)
res = []
for m in modes:
    kw = KW[m]
    info = sr.workspace_info(mask, cfg.B, cfg.H, cfg.S, cfg.D, sr.dtype_code(tdt), causal=cfg.causal,
                             tile_n=kw.get("tile_n", 0), fused=kw.get("fused", True))
    per = 4 * base[0].numel() * 2 + info["total_bytes"]
    n = max(2, min(8, math.ceil(2 * (126 << 20) / per)))
    sets = []
    for i in range(n):
        q, k, v = base if i == 0 else [x.clone() for x in base]
        o = torch.empty_like(q)
        ws = torch.empty(info["total_bytes"], dtype=torch.uint8, device=dev)
        sets.append((q, k, v, o, ws))
    fns = [(lambda s=s: sr.call(mask, s[0], s[1], s[2], out=s[3], workspace=s[4], scale=cfg.scale, causal=cfg.causal,
                                **kw)) for s in sets]
    for f in fns:
        f()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for i in range(K):
            fns[i % n]()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(5):
        torch.cuda._sleep(400000)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / K * 1e3)
    res.append(f"{os.path.basename(os.environ.get('SR_MHA_LIB', 'libsr_mha.so')):16s} C{idx} {m:12s} "
               f"median {statistics.median(ts):8.2f} us  min {min(ts):8.2f}")
    del sets, fns, g
    torch.cuda.empty_cache()
print("\n".join(res), flush=True)
