"""Determinism check: run a config's recomposed layer several times with the same inputs and report
which workspace intermediates (X', m', d', r') or outputs differ between runs (only valid regions)."""
import sys
import numpy as np
import torch
sys.path.insert(0, '.')
import paper_conf_iiswc_choilkha22_b200 as sr, workloads as W  # noqa
from bench import Layer  # noqa
idx, n = int(sys.argv[1]), int(sys.argv[2])
stages = int(sys.argv[3]) if len(sys.argv) > 3 else 0
cfg = W.config(idx)
L = Layer(cfg, torch.device("cuda", 0), cfg.idx, sr, torch)
tdt = {"f16": torch.float16, "bf16": torch.bfloat16, "f32": torch.float32}[cfg.dtype]
info = sr.workspace_info(L.mask, cfg.B, cfg.H, cfg.S, cfg.D, sr.dtype_code(tdt), causal=cfg.causal)
ws = L.ws[True]
ns = info["n_slots"]
def snap():
    g = lambda k, cnt, dt: ws[info[k]:info[k] + cnt * torch.tensor([], dtype=dt).element_size()].view(dt).clone()
    return {"X": g("off_xprime", ns * 128 * info["tile_n"], torch.int16), "m": g("off_mprime", ns * 128, torch.float32),
            "d": g("off_dprime", ns * 128, torch.float32), "r": g("off_rprime", ns * 128, torch.float32),
            "O": L.out.clone()}
L.run(); torch.cuda.synchronize()
ref = snap()
for k in range(n):
    ws.fill_(0x7f)  # poison: anything not rewritten shows up
    L.run(); torch.cuda.synchronize()
    cur = snap()
    diffs = {}
    for key in ref:
        a, b = ref[key], cur[key]
        if key in ("m", "d"):  # unwritten invalid halves are poisoned: compare where ref is finite & run1 wrote
            mask = torch.isfinite(a) & torch.isfinite(b)
            nd = int(((a != b) & mask).sum())
        elif key == "X":
            nd = -1  # invalid halves are not written; skip bitwise X compare here
        else:
            nd = int((a != b).sum())
        diffs[key] = nd
    print("run", k, diffs, flush=True)
