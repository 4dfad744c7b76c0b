"""Back-to-back layer time of some configs under the current process environment (for sweeps of the
runtime knobs SR_LPT_FIXED, SR_G1_PAIR, SR_X_KEEP, ...: one process per setting).
    SR_G1_PAIR=0 python tools/env_sweep.py 2,6"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Layer, back_to_back, rotation_sets  # noqa: E402

dev = torch.device("cuda", 0)
tag = " ".join(f"{k}={v}" for k, v in sorted(os.environ.items()) if k.startswith("SR_") and k != "SR_MHA_LIB") or "defaults"
for c in [int(x) for x in sys.argv[1].split(",")]:
    cfg = W.config(c)
    L = Layer(cfg, dev, cfg.idx, sr, torch, variants=False)
    sets, _ = rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=False)
    t = back_to_back(torch, [x.run for x in sets], 20, 5, reps=5)
    print(f"{tag:40s} C{c}: median {statistics.median(t) * 1e3:7.2f} us  min {min(t) * 1e3:7.2f}", flush=True)
    del L, sets
    torch.cuda.empty_cache()
