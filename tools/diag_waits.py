"""Per-warp mbarrier wait breakdown of GEMM1 / GEMM2 from the diagnostic build (-DSR_DIAG_WAITS).

    python -m paper_conf_iiswc_choilkha22_b200.build --define SR_DIAG_WAITS=1 --out paper_conf_iiswc_choilkha22_b200/libsr_diag.so
    SR_MHA_LIB=paper_conf_iiswc_choilkha22_b200/libsr_diag.so python tools/diag_waits.py CFG [variant] [reps]

Each kernel is launched alone (stage bits), so the counters belong to it.  Prints, per warp, its
mean lifetime per CTA (us at the sampled clock) and the share spent in each wait class:
  GEMM1  TMA w0: c0 q_empty c1 k_empty | MMA w1: c0 q_full c1 k_full c2 acc_empty | IR w3: c0 st_full
         epilogue: c0 acc_full c1 bulk-store smem reuse c2 st_empty; phases: c3 tcgen05.ld + release,
                   c7 staging wait, c4 mask/max/exp/sum, c5 pack/st.shared/bulk store, c6 statistics
  GEMM2  X' w0: c0 x_empty | MMA w1: c0 v_full c1 a_full c2 o_empty | stats w2: c0 st_empty
         V w3: c0 v_empty | GS w4-11: c0 x_full c1 a_empty c2 st_full | epilogue w12-15: c0 o_full
  concurrent (k_conc.cu): GEMM1 as above on warps 0-11 (MMA w1: c3 item_free), GEMM2 on warps 12-27
"""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import Layer  # noqa: E402

idx = int(sys.argv[1])
variant = sys.argv[2] if len(sys.argv) > 2 else "default"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
cfg = W.config(idx)
L = Layer(cfg, torch.device("cuda", 0), cfg.idx, sr, torch)
kw = {"fuse_ir": variant == "fuse_ir", "ir_kernel": variant == "ir_kernel", "two_kernels": variant == "two_kernels"}
lib = sr.lib()
KDW = 8
NW = 32
buf = (C.c_ulonglong * (NW * (KDW + 1)))()
L.run(**kw)
torch.cuda.synchronize()
ncta = 148
if variant == "concurrent":  # the concurrent kernel (k_conc.cu): GEMM1 warps 0-11, GEMM2 warps 12-27
    kw = {"concurrent": True}
    stages = (("CONC GEMM1", 0, lambda b: lib.sr_diag_read_conc(1, b)), ("CONC GEMM2", 0, lambda b: lib.sr_diag_read_conc(2, b)))
elif variant == "default":  # the one-launch kernel: phase 1 / phase 2 counters of k_fused.cu
    f1 = lambda b: lib.sr_diag_read_fused(1, b)
    f2 = lambda b: lib.sr_diag_read_fused(2, b)
    stages = (("PHASE1 (GEMM1)", 0, f1), ("PHASE2 (GEMM2)", 0, f2))
else:
    stages = (("GEMM1", 1, lib.sr_diag_read_g1), ("GEMM2", 4, lib.sr_diag_read_g2))
for name, bit, fn in stages:
    fn(buf)
    for _ in range(reps):
        L.run(stages=bit, **kw)
    torch.cuda.synchronize()
    fn(buf)
    a = np.array(buf[:], dtype=np.float64).reshape(NW, KDW + 1) / reps / ncta
    print(f"{name} C{idx} {variant}: per CTA per launch (us at 1.965 GHz); wait shares of lifetime")
    for w in range(NW):
        if a[w, KDW] == 0:
            continue
        life = a[w, KDW]
        sh = " ".join(f"c{c}={a[w, c] / life:5.1%}" for c in range(KDW) if a[w, c] > 0)
        print(f"  w{w:2d} life {life / 1965:7.2f} us  {sh}")
