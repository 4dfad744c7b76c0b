"""Per-CTA phase timeline of the one-launch kernel (diagnostic build -DSR_DIAG_PHASES):
    python -m paper_conf_iiswc_choilkha22_b200.build --define SR_DIAG_PHASES=1 --out paper_conf_iiswc_choilkha22_b200/libsr_ph.so
    SR_MHA_LIB=paper_conf_iiswc_choilkha22_b200/libsr_ph.so python tools/diag_phases.py CFG"""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import FLUSH_BYTES, Layer  # noqa: E402

cfg = W.config(int(sys.argv[1]))
dev = torch.device("cuda", 0)
L = Layer(cfg, dev, cfg.idx, sr, torch)
flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)
buf = (C.c_ulonglong * (1024 * 8))()
rows = []
for rep in range(5):
    flush.zero_()
    torch.cuda._sleep(400000)
    L.run()
    torch.cuda.synchronize()
    sr.lib().sr_diag_read_phases(buf)
    a = np.frombuffer(buf, dtype=np.uint64).reshape(1024, 8)[:148].astype(np.float64)
    t0 = a[:, 0].min()
    rows.append(a)
a = rows[-1]
t0 = a[:, 0].min()
start, pro, p1, p2, n = (a[:, 0] - t0) / 1e3, (a[:, 1] - a[:, 0]) / 1e3, (a[:, 2] - a[:, 1]) / 1e3, (a[:, 3] - a[:, 2]) / 1e3, a[:, 4]
end = (a[:, 3] - t0) / 1e3
q = lambda x: f"min {x.min():6.2f} mean {x.mean():6.2f} max {x.max():6.2f}"
print(f"C{cfg.idx}: CTA start offset (us) {q(start)}")
print(f"  prologue {q(pro)}\n  phase 1  {q(p1)}\n  phase 2  {q(p2)}\n  end      {q(end)}\n  items    {q(n)}")
i = int(np.argmax(end))
print(f"  last CTA {i}: start {start[i]:.2f} phase1 {p1[i]:.2f} phase2 {p2[i]:.2f} items {n[i]:.0f}")

tiles, smid = a[:, 5], a[:, 6]
print(f"  tiles    {q(tiles)}   corr(end, tiles) = {np.corrcoef(end, tiles)[0, 1]:.3f}   "
      f"corr(phase1, tiles) = {np.corrcoef(p1, tiles)[0, 1]:.3f}   corr(phase2, tiles) = {np.corrcoef(p2, tiles)[0, 1]:.3f}")
fit = np.polyfit(np.stack([tiles, n]).T @ [1, 0], end, 1)
print(f"  end ~ {fit[0]:.3f} us/tile * tiles + {fit[1]:.2f}; residual std {np.std(end - np.polyval(fit, tiles)):.2f} us")
die = smid >= 74
print(f"  by SM half (smid < 74 / >= 74): end mean {end[~die].mean():.2f} / {end[die].mean():.2f}, "
      f"us per tile {(end[~die] / tiles[~die]).mean():.3f} / {(end[die] / tiles[die]).mean():.3f}")
if len(sys.argv) > 2:
    np.savetxt(sys.argv[2], np.stack([np.arange(148), smid, n, tiles, p1, p2, end]).T, fmt="%.3f",
               header="cta smid items tiles phase1_us phase2_us end_us")
