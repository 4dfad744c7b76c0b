"""Helpers shared by the GPU parity tests: seeded inputs -> device tensors, oracle masks, and
read-back of workspace intermediates.  Inputs come from workloads (no method arithmetic)."""
import numpy as np

import oracle
import workloads as W

TORCH_DT = {"f32": "float32", "f16": "float16", "bf16": "bfloat16"}


def to_dev(arr_storage, dtype, device="cuda"):
    import torch
    if dtype == "bf16":
        t = torch.from_numpy(arr_storage.view(np.int16).copy()).view(torch.bfloat16)
    else:
        t = torch.from_numpy(np.ascontiguousarray(arr_storage))
    return t.to(device)


def qkv(B, H, S, D, dtype, seed=0):
    t = W.make_qkv(B, H, S, D, dtype, seed_base=seed)
    return t, to_dev(t.q_s, dtype), to_dev(t.k_s, dtype), to_dev(t.v_s, dtype)


def oracle_mask(kind, kv_len=None, causal=False, layout=None, window=0, n_global=0):
    return oracle.Mask(kind={"dense": "none", "block": "block", "window": "window"}[kind], kv_len=kv_len,
                       causal=causal, layout=layout, window=window, n_global=n_global)


def ws_view(ws, info, key, n, dtype):
    import torch
    off = info[key]
    return ws[off:off + n * torch.tensor([], dtype=dtype).element_size()].view(dtype)
