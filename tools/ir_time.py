"""The paper's standalone IR kernel (SR_IR_KERNEL) alone: K back-to-back launches (one CUDA graph,
PDL-chained, statistics L2-warm) and single L2-flushed calls, per config (SR_MHA_LIB picks the build).
    python tools/ir_time.py CFG[,CFG..]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402

dev = torch.device("cuda", 0)
flush = (torch.empty(bench.FLUSH_BYTES, dtype=torch.uint8, device=dev), torch.ones(bench.FLUSH_BYTES // 4, device=dev))
tag = os.path.basename(os.environ.get("SR_MHA_LIB", "libsr_mha.so"))
for idx in [int(x) for x in sys.argv[1].split(",")]:
    cfg = W.config(idx)
    L = bench.Layer(cfg, dev, seed_base=cfg.idx, sr=sr, torch=torch)
    L.run(ir_kernel=True)
    b2b = statistics.median(bench.back_to_back(torch, [lambda: L.run(ir_kernel=True, stages=2)], 20, 5)) * 1e3
    one = statistics.median(bench.timed(torch, lambda: L.run(ir_kernel=True, stages=2), 20, 3, flush)) * 1e3
    lay = statistics.median(bench.timed(torch, lambda: L.run(ir_kernel=True), 10, 3, flush)) * 1e3
    print(f"{tag} C{idx}: IR back to back {b2b:.2f} us, single L2-flushed {one:.2f} us, layer {lay:.1f} us "
          f"(share {one / lay:.3f})", flush=True)
    del L
    torch.cuda.empty_cache()
