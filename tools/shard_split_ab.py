"""One GPU's shard of a head-sharded layer (k ranks), default one-launch path vs SR_SPLIT_KV, back
to back with inputs larger than L2 (median of 5 regions).   python tools/shard_split_ab.py CFG K..."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Layer, back_to_back, make_shard, rotation_sets  # noqa: E402

c = int(sys.argv[1])
ks = [int(x) for x in sys.argv[2:]] or [1, 2, 4, 8]
cfg = W.config(c)
dev = torch.device("cuda", 0)
for k in ks:
    sh = make_shard(cfg, 0, k) if k > 1 else None
    L = Layer(cfg, dev, cfg.idx, sr, torch, shard=sh, variants=False)
    sets, _ = rotation_sets(cfg, dev, 0, sr, torch, L, 0, sh, variants=False)
    # split_kv needs its workspace layout (partial region): size every set's workspace for it
    for x in sets:
        info = sr.workspace_info(x.mask, x.B, x.H, cfg.S, cfg.D, x.in_dt, causal=cfg.causal, tile_n=0)
        if x.ws[True].numel() < info["total_bytes"]:
            x.ws[True] = torch.empty(info["total_bytes"], dtype=torch.uint8, device=dev)
    r = {}
    for name, kw in (("default", {}), ("split_kv", dict(split_kv=True))):
        fns = [(lambda x=x: sr.call(x.mask, x.dev["q"], x.dev["k"], x.dev["v"], out=x.out, workspace=x.ws[True],
                                    **x.kw, **kw)) for x in sets]
        r[name] = statistics.median(back_to_back(torch, fns, 20, 5, reps=5)) * 1e3
    print(f"C{c} k={k} heads={L.BH}: default {r['default']:8.2f} us, split_kv {r['split_kv']:8.2f} us", flush=True)
    del L, sets
    torch.cuda.empty_cache()
