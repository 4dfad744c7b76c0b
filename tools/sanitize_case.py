"""One small run of each forward path (and the training backward) for compute-sanitizer
(tools/sanitize.sh): C1 (fp32 SIMT), a reduced C2 (BERT padding, fp16, D=64), a reduced C3
(GPT-Neo causal, bf16, D=128), a small BigBird and Longformer layer; default one-launch kernel,
the unfused baseline and the variants.  Output checked against the fp64 oracle."""
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from tests.gpu_util import oracle_mask, qkv  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "all"
cases = [
    ("C1", "dense", 1, 1, 128, 64, "f32", dict()),
    ("C2s", "dense", 4, 2, 512, 64, "f16", dict(kv_len=[512, 300, 65, 1])),
    ("C3s", "dense", 1, 4, 1024, 128, "bf16", dict(causal=True)),
    ("C4s", "block", 1, 2, 1024, 64, "f16", dict(layout=W.bigbird_layout(2, 1024, 64))),
    ("C5s", "window", 1, 2, 1024, 64, "f16", dict(window=512, n_global=8)),
    # one BigBird head at S = 4096: global rows of 64 chunks take the unfused softmax's long-row launch
    ("C4l", "block", 1, 1, 4096, 64, "f16", dict(layout=W.bigbird_layout(1, 4096, 64))),
]
paths = [("default", {}), ("unfused", dict(fused=False)), ("ir_kernel", dict(ir_kernel=True)),
         ("sd", dict(sd=True)), ("two_kernels", dict(two_kernels=True)), ("concurrent", dict(concurrent=True)),
         ("split_kv", dict(split_kv=True))]
worst = 0.0
for name, kind, B, H, S, D, dt, kw in cases:
    t, q, k, v = qkv(B, H, S, D, dt, seed=5)
    scale = 1 / math.sqrt(D)
    kw = dict(kw)
    lay = kw.pop("layout", None)
    mask = {"dense": lambda: sr.dense_mask(kw.get("kv_len")), "block": lambda: sr.block_mask(lay),
            "window": lambda: sr.window_mask(kw.get("window", 0), kw.get("n_global", 0))}[kind]()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale,
                           oracle_mask(kind, kw.get("kv_len"), kw.get("causal", False), lay, kw.get("window", 0),
                                       kw.get("n_global", 0)))
    for pname, pkw in (paths if dt != "f32" else paths[:1]):
        if which != "all" and which != pname:
            continue
        o = sr.call(mask, q, k, v, scale=scale, causal=kw.get("causal", False), out_dtype=torch.float32, **pkw)
        torch.cuda.synchronize()
        e = float(np.abs(o.double().cpu().numpy() - ref).max())
        worst = max(worst, e)
        print(f"{name} {pname}: max err {e:.3g}", flush=True)
    if dt != "f32" and which in ("all", "train"):
        layer = sr.AttentionTrain(mask, causal=kw.get("causal", False), scale=scale)
        o = layer.forward(q, k, v)
        layer.backward(torch.ones_like(q))
        torch.cuda.synchronize()
        print(f"{name} train fwd+bwd ok", flush=True)
assert worst <= 1e-2, worst
del q, k, v, o
torch.cuda.synchronize()
torch.cuda.empty_cache()  # hand torch's cached segments back, so memcheck's leak report shows only real leaks
print("sanitize_case ok")
