"""SR_CONCURRENT vs the one-launch default: agreement and back-to-back timing on one box.

    python tools/conc_ab.py [configs, default 3,6] [K]

For each config: every element of the concurrent kernel's fp32 context against the one-launch
kernel's (same inputs), max |diff|; then back-to-back layers (CUDA graph of K calls over rotating
input/workspace sets larger than 2x L2), median of 5 regions, both paths, same power state."""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402

cfgs = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "3,6").split(",")]
K = int(sys.argv[2]) if len(sys.argv) > 2 else 20
dev = torch.device("cuda", 0)
for idx in cfgs:
    cfg = W.config(idx)
    L = bench.Layer(cfg, dev, seed_base=cfg.idx, sr=sr, torch=torch, variants=False)
    d = L.dev
    kw = dict(scale=cfg.scale, causal=cfg.causal, out_dtype=torch.float32, workspace=L.ws[True])
    o1 = sr.call(L.mask, d["q"], d["k"], d["v"], **kw)
    o2 = sr.call(L.mask, d["q"], d["k"], d["v"], concurrent=True, **kw)
    torch.cuda.synchronize()
    diff = (o1 - o2).abs().max().item()
    print(f"C{idx} {cfg.name}: max|conc - default| fp32 context = {diff:.3g}  (max|o| {o1.abs().max().item():.3g})",
          flush=True)
    sets, _ = bench.rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=False)
    res = {}
    for name, extra in (("default", {}), ("concurrent", {"concurrent": True}), ("default2", {}),
                        ("concurrent2", {"concurrent": True})):
        fns = [(lambda x=x, e=extra: sr.call(x.mask, x.dev["q"], x.dev["k"], x.dev["v"], out=x.out, workspace=x.ws[True],
                                             scale=cfg.scale, causal=cfg.causal, **e)) for x in sets]
        g = bench.steps_graph(torch, fns, K)
        for _ in range(3):
            g.replay()
        ms = [bench.region(torch, g, K, warm=g) for _ in range(5)]
        res[name] = statistics.median(ms) * 1e3
        del g
    print(f"C{idx}: " + "  ".join(f"{k} {v:.1f} us" for k, v in res.items()), flush=True)
    del sets, L
    torch.cuda.empty_cache()
