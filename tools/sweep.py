"""the paper's case-study axes (Fig. 9) on B200 --
sequence length L and batch size -- plus GPT-Neo's local-attention layers (window 256, causal) as a
second GPT-Neo workload (GPT-Neo alternates global and local attention).

For every point: attention layers/s of the default recomposed path (one launch: GEMM1+LS+IR then
GS+GEMM2 per CTA) and of the in-repo unfused baseline (GEMM1 -> row softmax -> GEMM2), each as one
L2-flushed call, the speedup, the algorithmic HBM
bytes of both, and a parity spot check of 48 sampled rows against the fp64 oracle (fp32 context,
tolerance 1e-2 as in tests/).  The paper reports whole-model speedups on A100 (context only); this
measures the attention layer itself.

    python tools/sweep.py [--out profiles/r1_sweep.json] [--quick]
"""
import argparse
import dataclasses
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402  (test infrastructure: parity spot checks only)
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402
from bench import FLUSH_BYTES, Layer, alg_bytes, alg_bytes_default, oracle_mask_for, timed  # noqa: E402


def points(quick):
    """(axis, model, Config) triples.  Base shapes are BASELINE.json's configs 2-5; the L sweep keeps
    each config's batch, the batch sweep each config's L (Fig. 9(a), 9(b))."""
    out = []
    Ls = [512, 1024, 2048, 4096] if not quick else [1024, 4096]
    Bs = [1, 2, 4, 8, 16] if not quick else [1, 8]
    bert, neo, bb, lf = (W.config(i) for i in (2, 3, 4, 5))

    def bert_at(S, B):  # padding pattern of C2 scaled to S (same fractions of the sequence)
        kv = [max(1, min(S, round(x * S / 512))) for x in bert.kv_len]
        kv = (kv * ((B + len(kv) - 1) // len(kv)))[:B]
        return dataclasses.replace(bert, idx=0, name=f"bert_L{S}_B{B}", S=S, B=B, kv_len=kv)

    neo_local = lambda S, B: dataclasses.replace(neo, idx=0, name=f"gptneo_local_L{S}_B{B}", kind="window", S=S, B=B,
                                                 window=510, n_global=0)
    for S in Ls:
        out.append(("L", "BERT", bert_at(S, bert.B)))
        out.append(("L", "GPT-Neo", dataclasses.replace(neo, idx=0, name=f"gptneo_L{S}", S=S)))
        out.append(("L", "GPT-Neo local", neo_local(S, neo.B)))
        if S >= 1024:
            out.append(("L", "BigBird", dataclasses.replace(bb, idx=0, name=f"bigbird_L{S}", S=S)))
            out.append(("L", "Longformer", dataclasses.replace(lf, idx=0, name=f"longformer_L{S}", S=S)))
    for B in Bs:
        out.append(("batch", "BERT", bert_at(bert.S, B)))
        out.append(("batch", "GPT-Neo", dataclasses.replace(neo, idx=0, name=f"gptneo_B{B}", B=B)))
        out.append(("batch", "GPT-Neo local", neo_local(neo.S, B)))
        out.append(("batch", "BigBird", dataclasses.replace(bb, idx=0, name=f"bigbird_B{B}", B=B)))
        out.append(("batch", "Longformer", dataclasses.replace(lf, idx=0, name=f"longformer_B{B}", B=B)))
    return out


def parity(L, cfg, n=48, seed=0):
    """Max |gpu - oracle| over n sampled rows (fp32 context of the same layer)."""
    t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=cfg.idx)
    o = sr.call(L.mask, L.dev["q"], L.dev["k"], L.dev["v"], out_dtype=torch.float32, tile_n=L.tile_n, **L.kw)
    torch.cuda.synchronize()
    rows = np.random.Generator(np.random.PCG64(seed)).integers(0, cfg.BH * cfg.S, size=n)
    ref = oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, oracle_mask_for(cfg))
    got = o.reshape(-1, cfg.D)[torch.from_numpy(rows).cuda()].double().cpu().numpy()
    return float(np.abs(got - ref).max())


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2_sweep.json"))
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--steps", type=int, default=10)
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    flush = (torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev),
             torch.ones(FLUSH_BYTES // 4, dtype=torch.float32, device=dev))
    res = []
    for axis, model, cfg in points(args.quick):
        L = Layer(cfg, dev, seed_base=cfg.idx, sr=sr, torch=torch)
        L.run()
        tr = statistics.mean(timed(torch, lambda: L.run(), args.steps, 3, flush))
        L.run(fused=False)
        tu = statistics.mean(timed(torch, lambda: L.run(fused=False), args.steps, 3, flush))
        rb = sum(alg_bytes_default(cfg, L.stored, L.T).values())
        ub = sum(alg_bytes(cfg, L.stored_u, L.Tu)[1].values())
        err = parity(L, cfg)
        e = {"axis": axis, "model": model, "name": cfg.name, "B": cfg.B, "H": cfg.H, "L": cfg.S, "D": cfg.D,
             "dtype": cfg.dtype, "layers_per_s": round(1e3 / tr, 1), "ms": round(tr, 4),
             "unfused_layers_per_s": round(1e3 / tu, 1), "speedup_vs_unfused": round(tu / tr, 3),
             "alg_bytes": int(rb), "alg_bytes_unfused": int(ub), "byte_reduction": round(1 - rb / ub, 4),
             "hbm_GBps": round(rb / (tr * 1e-3) / 1e9, 1), "max_abs_err_48_rows": err, "parity_ok": err <= 1e-2}
        print(json.dumps(e), flush=True)
        res.append(e)
        del L
        torch.cuda.empty_cache()
    json.dump({"what": __doc__.strip().splitlines()[0], "flush": "L2 flushed before every timed step",
               "points": res}, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
