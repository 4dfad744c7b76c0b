"""GPU parity of the training backward (§6 Eq. 3) against the fp64 backward
oracle (oracle/backward.py), element by element, through the C ABI (sr_mha_*_bwd) after the
default forward on the same SR_WS_TRAIN workspace.

Tolerance (DESIGN.md §Backward parity): with fp32 gradient outputs,
    max |g - g_ref| <= 1e-2 * max(1, max |g_ref|)          for g in dQ, dK, dV
-- the north star's 16-bit bound, scaled by the gradient's magnitude: every term of the three
contractions carries at most two roundings to the 16-bit MMA dtype (y and dS', relative 2^-9 for
bf16, 2^-12 for fp16) plus the fp16 X' (2^-12), so the error of a sum is below ~2^-8 of the sum of
its absolute terms.  Gradients stored in the 16-bit dtype add half an ulp of that dtype.
"""
import math

import numpy as np
import pytest

import workloads as W
from oracle import backward as OB
from tests.gpu_util import to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

TORCH = {"f16": torch.float16, "bf16": torch.bfloat16}


def _ulp_half(dtype, ref):
    mant = {"f16": 10, "bf16": 7}[dtype]
    e = np.floor(np.log2(np.maximum(np.abs(ref), 2.0 ** -14)))
    return 0.5 * 2.0 ** (e - mant)


def run_bwd(kind, B, H, S, D, dtype, *, causal=False, kv_len=None, layout=None, window=0, n_global=0, tile_n=0,
            seed=0, grads_f32=True, heads=None):
    t = W.make_qkv(B, H, S, D, dtype, seed_base=seed)
    do_s, do64 = W.make_dout(B, H, S, D, dtype, seed_base=seed)
    q, k, v, do = (to_dev(x, dtype) for x in (t.q_s, t.k_s, t.v_s, do_s))
    scale = 1 / math.sqrt(D)
    mask = {"dense": lambda: sr.dense_mask(kv_len), "block": lambda: sr.block_mask(layout),
            "window": lambda: sr.window_mask(window, n_global)}[kind]()
    layer = sr.AttentionTrain(mask, causal=causal, scale=scale, tile_n=tile_n)
    o = layer.forward(q, k, v, out_dtype=torch.float32 if grads_f32 else TORCH[dtype])
    dq, dk, dv = layer.backward(do)
    torch.cuda.synchronize()
    okw = {"dense": dict(kind="none", kv_len=kv_len), "block": dict(kind="block", layout=layout),
           "window": dict(kind="window", window=window, n_global=n_global)}[kind]
    ref = OB.attention_backward(t.q64, t.k64, t.v64, do64, scale, heads=heads, causal=causal, **okw)
    got = [x.float().cpu().numpy().astype(np.float64) for x in (o, dq, dk, dv)]
    if heads is not None:
        sel = [divmod(int(g), H) for g in heads]
        got = [np.stack([x[b, h] for b, h in sel]) for x in got]
        ref = [np.stack([x[b, h] for b, h in sel]) for x in ref]
    return got, ref


def check(got, ref, dtype, grads_f32=True, what=""):
    errs = {}
    for name, g, r in zip(("O", "dQ", "dK", "dV"), got, ref):
        assert np.isfinite(g).all(), f"{what} {name}: non-finite"
        err = np.abs(g - r)
        tol = (1e-2 if name == "O" else 1e-2 * max(1.0, float(np.abs(r).max())))
        if not grads_f32:
            tol = tol + _ulp_half(dtype, r)
        bad = err > tol
        assert not bad.any(), f"{what} {name}: {bad.sum()} over tolerance, max err {err.max():.3g} (max|ref| {np.abs(r).max():.3g})"
        errs[name] = float(err.max())
    return errs


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
@pytest.mark.parametrize("D", [64, 128])
def test_dense_causal_padding(dtype, D):
    got, ref = run_bwd("dense", 2, 2, 384, D, dtype, causal=True, kv_len=[384, 200], seed=1)
    check(got, ref, dtype, what=f"dense causal kv_len {dtype} D{D}")


@pytest.mark.parametrize("tile_n", [64, 128])
def test_dense_tile_widths(tile_n):
    got, ref = run_bwd("dense", 1, 3, 512, 64, "f16", kv_len=[449], tile_n=tile_n, seed=2)
    check(got, ref, "f16", what=f"dense T={tile_n}")


def test_dense_no_mask_bf16_stored_grads():
    got, ref = run_bwd("dense", 2, 2, 256, 128, "bf16", seed=3, grads_f32=False)
    check(got, ref, "bf16", grads_f32=False, what="dense bf16 stored grads")


def test_empty_rows_and_keys():
    # kv_len = 0: no kept key anywhere in batch 0 -> O = dQ = dK = dV = 0 there; batch 1 ragged
    got, ref = run_bwd("dense", 2, 1, 256, 64, "f16", kv_len=[0, 130], seed=4)
    check(got, ref, "f16", what="kv_len 0")
    for g in got:
        assert not g[0].any()


@pytest.mark.parametrize("causal", [False, True])
def test_blocksparse(causal):
    H, S = 2, 512
    lay = W.random_layout(H, S // 64, 64, 0.35, seed=5)
    got, ref = run_bwd("block", 1, H, S, 64, "f16", layout=lay, causal=causal, seed=5)
    check(got, ref, "f16", what=f"blocksparse causal={causal}")


def test_blocksparse_empty_block_rows():
    H, S = 1, 512
    nb = S // 64
    rows = [({0, r} if r % 3 else set()) for r in range(nb)]  # every third block-row empty
    lay = W.csr_from_sets(64, [rows])
    got, ref = run_bwd("block", 2, H, S, 64, "f16", layout=lay, seed=6)
    check(got, ref, "f16", what="blocksparse empty rows")


@pytest.mark.parametrize("causal", [False, True])
def test_window(causal):
    got, ref = run_bwd("window", 1, 2, 640, 64, "f16", window=128, n_global=8, causal=causal, seed=7)
    check(got, ref, "f16", what=f"window causal={causal}")


@pytest.mark.parametrize("idx", [2, 3, 4, 5])
def test_full_configs_every_head(idx):
    """BASELINE configs at full size, the launch configuration bench.py times; every head checked
    element by element against the oracle (O, dQ, dK, dV)."""
    cfg = W.config(idx)
    kw = dict(causal=cfg.causal, seed=cfg.idx)
    if cfg.kind == "dense":
        got, ref = run_bwd("dense", cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, kv_len=cfg.kv_len, **kw)
    elif cfg.kind == "blocksparse":
        got, ref = run_bwd("block", cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, layout=W.config_layout(cfg), **kw)
    else:
        got, ref = run_bwd("window", cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, window=cfg.window,
                           n_global=cfg.n_global, **kw)
    check(got, ref, cfg.dtype, what=f"C{idx}")


def test_backward_deterministic():
    outs = []
    for _ in range(2):
        got, _ = run_bwd("dense", 1, 2, 256, 64, "f16", causal=True, seed=8)
        outs.append(got)
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


def test_separate_dq_kernel():
    """SR_BWD_DQ_SEPARATE=1 (read once per process, so it runs in its own interpreter): dQ from its
    own kernel (the plain GEMM2 on dS' and K) instead of inside the dS' kernel."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = r"""
from tests.test_gpu_backward import run_bwd, check
import workloads as W
for kind, kw in (("dense", dict(B=2, H=2, S=384, D=64, dtype="f16", causal=True, kv_len=[384, 0])),
                 ("dense", dict(B=1, H=2, S=256, D=128, dtype="bf16")),
                 ("block", dict(B=1, H=2, S=512, D=64, dtype="f16", layout=W.random_layout(2, 8, 64, 0.35, seed=5)))):
    kw = dict(kw)
    B, H, S, D, dt = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    got, ref = run_bwd(kind, B, H, S, D, dt, **kw)
    check(got, ref, dt, what=kind)
print("ok")
"""
    env = dict(os.environ, SR_BWD_DQ_SEPARATE="1", PYTHONPATH=root)
    r = subprocess.run([sys.executable, "-c", script], cwd=root, env=env, capture_output=True, text=True, timeout=240)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]


@pytest.mark.parametrize("kind,kw", [
    ("dense", dict(B=2, H=2, S=192, D=64, dtype="f16", causal=True, kv_len=[192, 100])),
    ("dense", dict(B=1, H=3, S=320, D=128, dtype="bf16")),
    ("window", dict(B=1, H=2, S=448, D=64, dtype="f16", window=128, n_global=8)),
    ("block", dict(B=1, H=2, S=576, D=64, dtype="f16", layout="rand")),
], ids=lambda x: str(x)[:40] if isinstance(x, dict) else x)
def test_s_multiple_of_64(kind, kw):
    """S % 128 == 64: the last row-block / key column block is half inside the head; no gradient row
    of the next head is touched (every head compared in full)."""
    kw = dict(kw)
    if kw.get("layout") == "rand":
        kw["layout"] = W.random_layout(kw["H"], kw["S"] // 64, 64, 0.35, seed=12)
    B, H, S, D, dt = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    got, ref = run_bwd(kind, B, H, S, D, dt, seed=12, **kw)
    check(got, ref, dt, what=f"{kind} S={S}")
