"""Time a config's layer in several modes back to back (L2 flushed before every step):
    python tools/time_modes.py CFG [steps]   -> one line per mode, device ms per layer"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import FLUSH_BYTES, Layer, timed  # noqa: E402

idx = int(sys.argv[1])
K = int(sys.argv[2]) if len(sys.argv) > 2 else 30
cfg = W.config(idx)
dev = torch.device("cuda", 0)
flush = (torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev), torch.ones(FLUSH_BYTES // 4, device=dev))
L = Layer(cfg, dev, cfg.idx, sr, torch)
modes = {"default": {}, "gs_prologue": {"gs_prologue": True}, "two_kernels": {"two_kernels": True}, "fused_ir": {"fuse_ir": True},
         "ir_kernel": {"ir_kernel": True}, "g1_only": {"stages": 1, "two_kernels": True},
         "g2_only": {"stages": 4, "two_kernels": True}}
sel = os.environ.get("MODES")
if sel:
    modes = {k: v for k, v in modes.items() if k in sel.split(",")}
out = []
for rep in range(1):
    for name, kw in modes.items():
        if not os.environ.get("NO_DEFAULT"):  # (experiment builds whose one-launch kernel is not runnable)
            L.run()
        L.run(**{k_: v for k_, v in kw.items() if k_ != "stages"})  # uploads the schedule stage runs reuse
        ms = statistics.median(timed(torch, lambda: L.run(**kw), K, 3, flush))
        out.append(f"{os.environ.get('TAG', '')} C{idx} rep{rep} {name:10s} {ms * 1e3:8.2f} us")
print("\n".join(out))
