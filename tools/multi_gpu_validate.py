"""Multi-GPU validation: one layer of a BASELINE config sharded by heads across
ranks (paper_conf_iiswc_choilkha22_b200.shard), each rank runs its shard through the C ABI on its
GPU, the output shards are gathered over NCCL (the only collective, validation only), and rank 0
checks sampled rows against the fp64 oracle.

  python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 tools/multi_gpu_validate.py [--config 3]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import oracle  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_iiswc_choilkha22_b200 import shard as SH  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--rows", type=int, default=256)
    a = ap.parse_args()
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    lr = int(os.environ.get("LOCAL_RANK", 0))
    # SR_BENCH_SHARED_GPU=1: every rank on cuda:0 and the gather over gloo on host copies (a functional
    # check of the sharded layer's assembly on a one-GPU box)
    shared = os.environ.get("SR_BENCH_SHARED_GPU") == "1"
    if shared:
        lr = 0
    torch.cuda.set_device(lr)
    if shared:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=torch.device("cuda", lr))
    cfg = W.config(a.config)
    t = W.config_tensors(cfg)
    lay = W.config_layout(cfg)
    sh = SH.make_shard(rank, world, cfg.B, cfg.H, cfg.S, kv_len=cfg.kv_len, layout=lay)
    tdt = {"f16": torch.float16, "bf16": torch.bfloat16, "f32": torch.float32}[cfg.dtype]

    def dev(x):
        if cfg.dtype == "bf16":
            x = torch.from_numpy(x.view(np.int16).copy()).view(torch.bfloat16)
        else:
            x = torch.from_numpy(np.ascontiguousarray(x))
        return SH.shard_view(x, sh).contiguous().cuda()

    q, k, v = dev(t.q_s), dev(t.k_s), dev(t.v_s)
    kw = dict(scale=cfg.scale, causal=cfg.causal, out_dtype=torch.float32)
    if cfg.kind == "dense":
        o = sr.mha_dense(q, k, v, kv_len=sh.kv_len, **kw)
    elif cfg.kind == "blocksparse":
        o = sr.mha_blocksparse(q, k, v, sh.layout, **kw)
    else:
        o = sr.mha_sliding_window(q, k, v, cfg.window, cfg.n_global, **kw)
    # gather variable-size shards: pad to the largest, all_gather_into_tensor, trim on rank 0
    cdev = "cpu" if shared else "cuda"
    n = torch.tensor([sh.n], device=cdev)
    ns = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(ns, n)
    n_max = int(max(x.item() for x in ns))
    buf = torch.zeros(n_max, cfg.S, cfg.D, device=cdev)
    buf[:sh.n] = o.reshape(sh.n, cfg.S, cfg.D).to(cdev)
    if shared:
        parts = [torch.empty_like(buf) for _ in range(world)]
        dist.all_gather(parts, buf)
        allb = torch.cat(parts).cuda()
    else:
        allb = torch.empty(world * n_max, cfg.S, cfg.D, device="cuda")
        dist.all_gather_into_tensor(allb, buf)
    if rank == 0:
        full = torch.cat([allb[r * n_max:r * n_max + int(ns[r].item())] for r in range(world)]).reshape(-1, cfg.D)
        rng = np.random.Generator(np.random.PCG64(0))
        rows = np.sort(rng.choice(cfg.BH * cfg.S, size=a.rows, replace=False))
        m = (oracle.Mask(kind="block", layout=lay) if lay is not None else
             oracle.Mask(kind="window", window=cfg.window, n_global=cfg.n_global) if cfg.kind == "window" else
             oracle.Mask(kv_len=cfg.kv_len, causal=cfg.causal))
        ref = oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, m)
        err = float(np.abs(full[torch.from_numpy(rows).cuda()].double().cpu().numpy() - ref).max())
        print(f"multi_gpu_validate: C{cfg.idx} world={world} shards={[int(x.item()) for x in ns]} "
              f"max|err| over {a.rows} rows = {err:.3g} -> {'OK' if err <= 1e-2 else 'FAIL'}", flush=True)
        assert err <= 1e-2
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
