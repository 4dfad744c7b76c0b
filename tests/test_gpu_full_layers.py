"""GPU parity at the BASELINE configs' FULL sizes, every output row, every path.

The paper's claim is an identical result ("mathematically has a result identical to
that of the original softmax layer"), over every block layout (L177-L181).  So each test here runs
one whole layer of a BASELINE config (C2-C5, plus GPT-Neo's local-attention layer, SURVEY NEXT-3,
PAPER.md L185) in the launch configuration bench.py times, and compares EVERY element of the
context with the fp64 oracle's whole-layer output (``oracle.attention``, computed once per config):

  * fp32-accumulated context (out_dtype = float32): max |gpu - oracle| <= 1e-2    (north star)
  * stored in the config dtype: <= 1e-2 + half an ulp of that dtype at |o|        (reading R17)

Paths: the default one-launch kernel, the unfused baseline, and every variant (two launches, IR in
GEMM2, the paper's standalone IR kernel, SD, GS in the prologue).  Max errors are appended to
$SR_PARITY_REPORT (JSON lines) when that variable is set, so the GPU run keeps the numbers.
"""
import json
import os

import numpy as np
import pytest

import oracle
import workloads as W
from tests.gpu_util import to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

TORCH = {"f16": torch.float16, "bf16": torch.bfloat16}
CFGS = [2, 3, 4, 5, 6]  # 6 = GPT-Neo local attention (workloads.GPTNEO_LOCAL)

_cache = {}


def _ulp_half(dtype, ref):
    mant = {"f16": 10, "bf16": 7}[dtype]
    e = np.floor(np.log2(np.maximum(np.abs(ref), 2.0 ** -14)))
    return 0.5 * 2.0 ** (e - mant)


def report(**kw):
    path = os.environ.get("SR_PARITY_REPORT")
    if path:
        with open(path, "a") as f:
            f.write(json.dumps(kw) + "\n")


def oracle_mask(cfg):
    if cfg.kind == "dense":
        return oracle.Mask(kv_len=cfg.kv_len, causal=cfg.causal)
    if cfg.kind == "blocksparse":
        return oracle.Mask(kind="block", layout=W.config_layout(cfg), causal=cfg.causal)
    return oracle.Mask(kind="window", window=cfg.window, n_global=cfg.n_global, causal=cfg.causal)


def sr_mask(cfg):
    if cfg.kind == "dense":
        return sr.dense_mask(cfg.kv_len)
    if cfg.kind == "blocksparse":
        return sr.block_mask(W.config_layout(cfg))
    return sr.window_mask(cfg.window, cfg.n_global)


def layer(idx):
    """(cfg, device q/k/v, fp64 oracle output of the whole layer), computed once per config."""
    if idx not in _cache:
        cfg = W.config(idx)
        t = W.config_tensors(cfg)
        ref = oracle.attention(t.q64, t.k64, t.v64, cfg.scale, oracle_mask(cfg))
        dev = tuple(to_dev(x, cfg.dtype) for x in (t.q_s, t.k_s, t.v_s))
        _cache[idx] = (cfg, dev, ref)
    return _cache[idx]


VARIANTS = {
    # name: call keywords (tile_n as bench.py runs it)
    "default": dict(),
    "unfused": dict(fused=False),
    "two_kernels": dict(two_kernels=True, tile_n=128),
    "fuse_ir": dict(fuse_ir=True, tile_n=128),
    "ir_kernel": dict(ir_kernel=True, tile_n=128),
    "sd": dict(sd=True),
    "gs_prologue": dict(gs_prologue=True),
    "split_kv": dict(split_kv=True),
    "concurrent": dict(concurrent=True),
}


def run(cfg, dev, variant, out_dtype):
    kw = dict(VARIANTS[variant])
    if cfg.kind == "blocksparse" and kw.get("tile_n") == 128:
        kw["tile_n"] = 64  # block-sparse sub-vectors are the 64-key blocks
    q, k, v = dev
    o = sr.call(sr_mask(cfg), q, k, v, scale=cfg.scale, causal=cfg.causal, out_dtype=out_dtype, **kw)
    torch.cuda.synchronize()
    return o.double().cpu().numpy()


def compare(o, ref, dtype, stored, what):
    assert np.isfinite(o).all(), f"{what}: non-finite output"
    err = np.abs(o - ref)
    tol = 1e-2 + (_ulp_half(dtype, ref) if stored else 0.0)
    bad = err > tol
    emax = float(err.max())
    report(test=what, max_abs_err=emax, elements=int(err.size), over=int(bad.sum()),
           bound="1e-2 + ulp/2" if stored else "1e-2")
    assert not bad.any(), f"{what}: {bad.sum()} of {err.size} elements over tolerance, max err {emax:.4g}"
    return emax


@pytest.mark.parametrize("variant", list(VARIANTS))
@pytest.mark.parametrize("idx", CFGS)
def test_full_layer_every_row(idx, variant):
    """Every row of the layer, fp32-accumulated context vs the fp64 oracle (<= 1e-2)."""
    cfg, dev, ref = layer(idx)
    o = run(cfg, dev, variant, torch.float32)
    compare(o, ref, cfg.dtype, False, f"C{idx} {variant} fp32-context")


@pytest.mark.parametrize("idx", CFGS)
def test_full_layer_stored_dtype(idx):
    """Every row, output stored in the config dtype (the bench's launch configuration), against
    1e-2 + half an ulp (reading R17: C3 bf16 is predicted at 0.0101-0.0122, above 1e-2 and inside
    the half-ulp allowance -- the bf16 half-ulp is 0.0078 on [2, 4))."""
    cfg, dev, ref = layer(idx)
    o = run(cfg, dev, "default", TORCH[cfg.dtype])
    emax = compare(o, ref, cfg.dtype, True, f"C{idx} default stored-{cfg.dtype}")
    print(f"C{idx} stored {cfg.dtype}: max |o - oracle| = {emax:.5f}")


@pytest.mark.parametrize("idx", [2, 5])
def test_full_layer_unfused_stored_dtype(idx):
    cfg, dev, ref = layer(idx)
    o = run(cfg, dev, "unfused", TORCH[cfg.dtype])
    compare(o, ref, cfg.dtype, True, f"C{idx} unfused stored-{cfg.dtype}")
