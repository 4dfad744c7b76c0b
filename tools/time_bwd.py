"""Device time of the training backward per stage (L2 flushed before each step):
    python tools/time_bwd.py CFG [steps]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import FLUSH_BYTES, Layer, timed  # noqa: E402

idx = int(sys.argv[1])
K = int(sys.argv[2]) if len(sys.argv) > 2 else 20
cfg = W.config(idx)
dev = torch.device("cuda", 0)
flush = (torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev), torch.ones(FLUSH_BYTES // 4, device=dev))
L = Layer(cfg, dev, cfg.idx, sr, torch)
L.setup_train(cfg.idx)
L.train_step()
res = {"fwd": statistics.median(timed(torch, L.fwd_train, K, 3, flush)),
       "bwd": statistics.median(timed(torch, L.bwd, K, 3, flush))}
for name, st in (("prep_ds_dq", 1), ("dq_separate", 2), ("dk_dv", 4)):
    res[name] = statistics.median(timed(torch, lambda: L.bwd(stages=st), K, 3, flush))
print(os.environ.get("TAG", ""), f"C{idx}", " ".join(f"{k}={v * 1e3:.1f}us" for k, v in res.items()))
