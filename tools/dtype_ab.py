"""The C3 layer in bf16 vs fp16 inputs (same shape and mask), one-launch default, back to back.
    python tools/dtype_ab.py"""
import math
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

dev = torch.device("cuda", 0)
K, B, H, S, D = 20, 4, 16, 2048, 128
mask = sr.dense_mask(None)
for dt in (torch.bfloat16, torch.float16, torch.bfloat16, torch.float16):
    info = sr.workspace_info(mask, B, H, S, D, sr.dtype_code(dt), causal=True, tile_n=0)
    n = max(2, math.ceil(2 * (126 << 20) / (4 * B * H * S * D * 2 + info["total_bytes"])))
    sets = []
    for i in range(n):
        g = torch.Generator(device=dev).manual_seed(i)
        q, k, v = (torch.randn(B, H, S, D, device=dev, generator=g).to(dt) for _ in range(3))
        sets.append((q, k, v, torch.empty_like(q), torch.empty(info["total_bytes"], dtype=torch.uint8, device=dev)))
    res = {}
    for name, extra in (("default", {}), ("gs_prologue", {"gs_prologue": True})):
        fns = [(lambda s=s, e=extra: sr.call(mask, s[0], s[1], s[2], out=s[3], workspace=s[4], scale=D ** -0.5,
                                             causal=True, **e)) for s in sets]
        gr = bench.steps_graph(torch, fns, K)
        for _ in range(3):
            gr.replay()
        res[name] = statistics.median([bench.region(torch, gr, K, warm=gr) for _ in range(5)]) * 1e3
    print(dt, {k: round(v, 1) for k, v in res.items()}, flush=True)
    del sets, gr
    torch.cuda.empty_cache()
