"""Headline method A/B: K back-to-back layers of a config with the schedule uploaded by every call
(the bench headline) vs resident (SR_SCHED_RESIDENT), alternating regions in one process, plus the
same with 4 rotation sets.   python tools/headline_ab.py [CFG] [K]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Layer, region, rotation_sets, steps_graph  # noqa: E402

c = int(sys.argv[1]) if len(sys.argv) > 1 else 3
K = int(sys.argv[2]) if len(sys.argv) > 2 else 20
cfg = W.config(c)
dev = torch.device("cuda", 0)
L = Layer(cfg, dev, cfg.idx, sr, torch, variants=False)
sets, _ = rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=False)
extra = [Layer(cfg, dev, cfg.idx + 500 + i, sr, torch, variants=False) for i in range(2)]
graphs = {
    "upload": steps_graph(torch, [x.run for x in sets], K),
    "resident": steps_graph(torch, [(lambda x=x: x.run(resident=True)) for x in sets], K),
    "upload_4sets": steps_graph(torch, [x.run for x in sets + extra], K),
    "resident_4sets": steps_graph(torch, [(lambda x=x: x.run(resident=True)) for x in sets + extra], K),
}
res = {k: [] for k in graphs}
for rep in range(6):
    for k, g in graphs.items():
        torch.cuda.synchronize()
        res[k].append(region(torch, g, K, warm=g))
for k, v in res.items():
    print(f"C{c} {k:15s} sets={len(sets) if '4' not in k else len(sets) + 2}: median {statistics.median(v) * 1e3:8.2f} us  "
          f"min {min(v) * 1e3:8.2f}  max {max(v) * 1e3:8.2f}")
