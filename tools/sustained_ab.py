"""Sustained-load timing of one library build (SR_MHA_LIB): K back-to-back layers replayed for
`secs` seconds (the clock settles under the 1 kW power cap), then 5 regions; prints the median layer
time, and the SM clock / power nvidia-smi saw meanwhile.   python tools/sustained_ab.py CFG [secs]"""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Clocks, Layer, region, rotation_sets, steps_graph  # noqa: E402

c = int(sys.argv[1]) if len(sys.argv) > 1 else 3
secs = float(sys.argv[2]) if len(sys.argv) > 2 else 2.0
cfg = W.config(c)
dev = torch.device("cuda", 0)
L = Layer(cfg, dev, cfg.idx, sr, torch, variants=False)
sets, _ = rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=False)
g = steps_graph(torch, [x.run for x in sets], 20)
cold = region(torch, g, 20, warm=g)
clk = Clocks(os.environ.get("CUDA_VISIBLE_DEVICES", "0").split(",")[0])
clk.start()
t_end = time.perf_counter() + secs
while time.perf_counter() < t_end:
    g.replay()
torch.cuda.synchronize()
v = [region(torch, g, 20, warm=g) for _ in range(5)]
info = clk.stop()
print(f"{os.path.basename(os.environ.get('SR_MHA_LIB', 'libsr_mha.so')):16s} C{c}: first region {cold * 1e3:7.2f} us, "
      f"sustained median {statistics.median(v) * 1e3:7.2f} us (min {min(v) * 1e3:.2f}), clocks {info}", flush=True)
