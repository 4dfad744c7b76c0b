"""Where SR_CONCURRENT beats the one-launch kernel (D = 128, bf16): back-to-back layer time over
causal dense and causal-window shapes of GPT-Neo's head geometry.
    python tools/conc_sweep.py"""
import math
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

dev = torch.device("cuda", 0)
K = 20
cases = [("causal", 4, 16, S, None) for S in (512, 1024, 1536, 2048, 4096)] + \
        [("window", 4, 16, S, w) for S in (2048, 4096) for w in (254, 510, 1022)]
for kind, B, H, S, w in cases:
    D = 128
    mask = sr.dense_mask(None) if kind == "causal" else sr.window_mask(w, 0)
    st = sr.schedule_stats(mask, B, H, S, causal=True, tile_n=64)
    info = sr.workspace_info(mask, B, H, S, D, sr.dtype_code(torch.bfloat16), causal=True, tile_n=0)
    per = 4 * B * H * S * D * 2 + info["total_bytes"]
    n = max(2, min(8, math.ceil(2 * (126 << 20) / per)))
    sets = []
    for i in range(n):
        g = torch.Generator(device=dev).manual_seed(i)
        q, k, v = (torch.randn(B, H, S, D, device=dev, generator=g).to(torch.bfloat16) for _ in range(3))
        sets.append((q, k, v, torch.empty_like(q), torch.empty(info["total_bytes"], dtype=torch.uint8, device=dev)))
    res = {}
    for name, extra in (("default", {}), ("conc", {"concurrent": True})):
        fns = [(lambda s=s, e=extra: sr.call(mask, s[0], s[1], s[2], out=s[3], workspace=s[4], scale=D ** -0.5,
                                             causal=True, **e)) for s in sets]
        gr = bench.steps_graph(torch, fns, K)
        for _ in range(3):
            gr.replay()
        res[name] = statistics.median([bench.region(torch, gr, K, warm=gr) for _ in range(5)]) * 1e3
        del gr
    print(f"{kind:6s} S={S:5d} w={w} tiles={st[0]} per-item={st[0] / (B * H * S / 128):.1f}: "
          f"default {res['default']:.1f} us  conc {res['conc']:.1f} us  ratio {res['conc'] / res['default']:.3f}",
          flush=True)
    del sets
    torch.cuda.empty_cache()
