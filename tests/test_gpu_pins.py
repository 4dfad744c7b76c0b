"""SURVEY §8(c) pins driven THROUGH the tensor-core path.

  P3 (dtypes)  closed form at GPU shapes, fp16 / bf16, D = 64 / 128, dense and causal, every path:
               q_i = c e_i, k_i = v_i = e_i for i < 4, zero rows elsewhere, c = 1 (exact in every
               dtype) and a = e^{c * scale} in place of the 3 of P3 (SURVEY §8(c) P3 "dtypes").
  P7 (nb = 3)  every block layout of 3 block-rows x 3 block-columns with no empty row (7^3 = 343),
               all in one call (layout_heads = 343), embedded in S = 256 two ways so that both
               64-row pairings of the 128-row tiles see every combination; vs the fp64 oracle.
  P7 (window)  window in {0, 2, 126, 128, 130, 254} x n_global in {0, 1, 8, 64} x causal, S = 256.

Cites: PAPER.md L131 (identical result), L177-L181 (block-sparse / window layouts), L51-L58.
"""
import itertools
import math

import numpy as np
import pytest

import oracle
import workloads as W
from tests.gpu_util import oracle_mask, qkv, to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

TORCH = {"f16": torch.float16, "bf16": torch.bfloat16}
PATHS = {"default": {}, "unfused": dict(fused=False), "two_kernels": dict(two_kernels=True, tile_n=128),
         "fuse_ir": dict(fuse_ir=True, tile_n=128), "ir_kernel": dict(ir_kernel=True, tile_n=128),
         "sd": dict(sd=True), "gs_prologue": dict(gs_prologue=True)}


# ------------------------------------------------------------------------------------------ P3

def p3_closed_form(S, D, scale, causal, c=1.0):
    """SURVEY §8(c) P3 with a = e^{c*scale}: rows i < 4 see one score c*scale (key i) and zeros."""
    a = math.exp(c * scale)
    want = np.zeros((S, D))
    for i in range(S):
        n_keys = (i + 1) if causal else S  # keys the row keeps
        for col in range(4):
            if causal and col > i:
                continue
            if i < 4:
                want[i, col] = (a if col == i else 1.0) / (a + n_keys - 1)
            else:
                want[i, col] = 1.0 / n_keys
    return want


@pytest.mark.parametrize("path", list(PATHS))
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("dtype,D", [("f16", 64), ("bf16", 64), ("f16", 128), ("bf16", 128)])
def test_p3_dtypes_closed_form(dtype, D, causal, path):
    S, H = 384, 2
    q = torch.zeros(1, H, S, D, dtype=TORCH[dtype])
    k = torch.zeros(1, H, S, D, dtype=TORCH[dtype])
    for i in range(4):
        q[0, :, i, i] = 1.0
        k[0, :, i, i] = 1.0
    q, k = q.cuda(), k.cuda()
    v = k.clone()
    scale = 1 / math.sqrt(D)
    o = sr.call(sr.dense_mask(None), q, k, v, scale=scale, causal=causal, out_dtype=torch.float32,
                **PATHS[path]).double().cpu().numpy()
    want = p3_closed_form(S, D, scale, causal)
    # every output element is ONE product Y_ic * 1 (v_j = e_j): its error is the roundings of X'
    # (fp16, 2^-11 relative) and of Y to the MMA dtype (2^-9 bf16, 2^-11 fp16) -- bound 2^-8 relative
    for h in range(H):
        np.testing.assert_allclose(o[0, h], want, rtol=2.0 ** -8, atol=1e-7, err_msg=f"{path} head {h}")


# ------------------------------------------------------------------------------------------ P7 nb=3

def _layouts_nb3():
    opts = [c for r in (1, 2, 3) for c in itertools.combinations(range(3), r)]  # 7 non-empty rows
    return list(itertools.product(opts, repeat=3))  # 343


def _embed(lays, shift):
    """Embed 3x3 layouts into nb = 4: shift 0 -> rows/cols 0-2 (row 3 = {3}); shift 1 -> rows/cols
    1-3 (row 0 = {0}).  Block-rows (0, 1) and (2, 3) share a 128-row tile."""
    heads = []
    for rows in lays:
        r = [set(c + shift for c in row) for row in rows]
        heads.append(r + [{3}] if shift == 0 else [{0}] + r)
    return W.csr_from_sets(64, heads)


@pytest.mark.parametrize("path", ["default", "unfused", "ir_kernel", "sd"])
@pytest.mark.parametrize("shift,causal", [(0, False), (1, False), (0, True)])
def test_all_block_layouts_nb3(shift, causal, path):
    lays = _layouts_nb3()
    assert len(lays) == 343
    lay = _embed(lays, shift)
    H, S, D = len(lays), 256, 64
    t, q, k, v = qkv(1, H, S, D, "f16", seed=11 + shift)
    scale = 1 / math.sqrt(D)
    kw = dict(PATHS[path])
    if kw.get("tile_n") == 128:
        kw["tile_n"] = 64  # block-sparse sub-vectors are the 64-key blocks
    o = sr.call(sr.block_mask(lay), q, k, v, scale=scale, causal=causal, out_dtype=torch.float32,
                **kw).double().cpu().numpy()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale, oracle_mask("block", None, causal, lay))
    err = np.abs(o - ref)
    assert np.isfinite(o).all()
    bad = np.argwhere(err > 1e-2)
    assert bad.size == 0, f"{len(bad)} elements over 1e-2 (first: head {bad[0][1]} layout {lays[bad[0][1]]})"


# ------------------------------------------------------------------------------------------ P7 window

@pytest.mark.parametrize("path", ["default", "unfused"])
@pytest.mark.parametrize("causal", [False, True])
@pytest.mark.parametrize("n_global", [0, 1, 8, 64])
@pytest.mark.parametrize("window", [0, 2, 126, 128, 130, 254])
def test_window_grid(window, n_global, causal, path):
    B, H, S, D = 1, 2, 256, 64
    t, q, k, v = qkv(B, H, S, D, "f16", seed=window + n_global)
    scale = 1 / math.sqrt(D)
    o = sr.call(sr.window_mask(window, n_global), q, k, v, scale=scale, causal=causal,
                out_dtype=torch.float32, **PATHS[path]).double().cpu().numpy()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale, oracle_mask("window", None, causal, None, window, n_global))
    assert np.abs(o - ref).max() <= 1e-2


# ------------------------------------------------------------------------------------------ GPT-Neo local

@pytest.mark.parametrize("path", ["default", "unfused", "two_kernels"])
def test_gptneo_local_small(path):
    """GPT-Neo local attention (window 256 -> keys i-255..i), bf16, D = 128, causal,
    at a smaller S than the full config (which test_gpu_full_layers covers)."""
    B, H, S, D = 2, 2, 1024, 128
    t, q, k, v = qkv(B, H, S, D, "bf16", seed=21)
    scale = 1 / math.sqrt(D)
    o = sr.call(sr.window_mask(510, 0), q, k, v, scale=scale, causal=True, out_dtype=torch.float32,
                **PATHS[path]).double().cpu().numpy()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale, oracle_mask("window", None, True, None, 510, 0))
    assert np.abs(o - ref).max() <= 1e-2
