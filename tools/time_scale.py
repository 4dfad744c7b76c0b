"""Per-kernel device time vs batch size for one config (fixed vs marginal cost):
    python tools/time_scale.py CFG B1 B2 ..."""
import dataclasses
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import FLUSH_BYTES, Layer, timed  # noqa: E402

cfg0 = W.config(int(sys.argv[1]))
dev = torch.device("cuda", 0)
flush = (torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev), torch.ones(FLUSH_BYTES // 4, device=dev))
for b in sys.argv[2:]:
    B = int(b)
    kv = None if cfg0.kv_len is None else (cfg0.kv_len * ((B + 7) // 8))[:B]
    cfg = dataclasses.replace(cfg0, B=B, kv_len=kv)
    L = Layer(cfg, dev, cfg.idx, sr, torch)
    L.run()
    t = {n: statistics.median(timed(torch, lambda s=s: L.run(stages=s), 20, 3, flush)) for n, s in
         (("chain", 0), ("g1", 1), ("g2", 4))}
    print(f"{os.environ.get('TAG', '')} C{cfg.idx} B={B} " + " ".join(f"{k}={v * 1e3:.2f}us" for k, v in t.items()), flush=True)
