"""Time SR_CONCURRENT and the one-launch default back to back (same process; SR_MHA_LIB picks the build).
    python tools/conc_time.py CFG[,CFG..] [K]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402

K = int(sys.argv[2]) if len(sys.argv) > 2 else 20
dev = torch.device("cuda", 0)
tag = os.path.basename(os.environ.get("SR_MHA_LIB", "libsr_mha.so"))
for idx in [int(x) for x in sys.argv[1].split(",")]:
    cfg = W.config(idx)
    L = bench.Layer(cfg, dev, seed_base=cfg.idx, sr=sr, torch=torch, variants=False)
    sets, _ = bench.rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=False)
    res = {}
    for name, extra in (("default", {}), ("conc", {"concurrent": True})):
        fns = [(lambda x=x, e=extra: x.run(**e)) for x in sets]
        g = bench.steps_graph(torch, fns, K)
        for _ in range(3):
            g.replay()
        res[name] = statistics.median([bench.region(torch, g, K, warm=g) for _ in range(5)]) * 1e3
        del g
    print(f"{tag} C{idx}: " + "  ".join(f"{k} {v:.1f} us" for k, v in res.items()), flush=True)
    del sets, L
    torch.cuda.empty_cache()
