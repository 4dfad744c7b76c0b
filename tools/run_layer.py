"""Run one config's layer a few times (for ncu captures):
    python tools/run_layer.py CFG [fused|unfused|two_kernels|fused_ir|ir_kernel|sd|conc|train] [reps]
(train: forward + training backward on an SR_WS_TRAIN workspace)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Layer  # noqa: E402

idx = int(sys.argv[1])
mode = sys.argv[2] if len(sys.argv) > 2 else "fused"
fused = mode != "unfused"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
cfg = W.config(idx)
L = Layer(cfg, torch.device("cuda", 0), cfg.idx, sr, torch)
if mode == "train":
    L.setup_train(cfg.idx)
for _ in range(reps):
    if mode == "train":
        L.train_step()
    else:
        L.run(fused=fused, fuse_ir=mode == "fused_ir", sd=mode == "sd", ir_kernel=mode == "ir_kernel",
              two_kernels=mode == "two_kernels", concurrent=mode == "conc")
torch.cuda.synchronize()
print("ok", cfg.name, mode)
