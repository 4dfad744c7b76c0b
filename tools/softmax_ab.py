"""The unfused baseline's softmax launch(es) alone, back to back over rotating sets, per config.
    python tools/softmax_ab.py CFG[,CFG..]   (SR_SOFTMAX_RSPLIT etc. from the environment)"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402

dev = torch.device("cuda", 0)
for idx in [int(x) for x in sys.argv[1].split(",")]:
    cfg = W.config(idx)
    L = bench.Layer(cfg, dev, seed_base=cfg.idx, sr=sr, torch=torch, variants=False)
    sets, _ = bench.rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=False)
    for x in sets:
        x.run(fused=False)
    t = statistics.median(bench.back_to_back(torch, [(lambda x=x: x.run(fused=False, stages=2)) for x in sets], 20, 5))
    nb = bench.alg_bytes(cfg, L.stored_u, 64)[1]["softmax"]
    print(f"rsplit={os.environ.get('SR_SOFTMAX_RSPLIT', '-')} C{idx}: softmax {t * 1e3:.1f} us, "
          f"{nb / (t * 1e-3) / 1e9:.0f} GB/s", flush=True)
    del sets, L
    torch.cuda.empty_cache()
