"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle, element by element.

Tolerances (BASELINE.json north_star):
  fp32 mode (SIMT):                       max |gpu - oracle| <= 1e-5
  fp16 / bf16, fp32-accumulated context:  max |gpu - oracle| <= 1e-2   (out_dtype = float32)
  fp16 / bf16 stored output:              <= 1e-2 + half an ulp of the output dtype at |o|
Small cases span several tiles and ragged (masked) tails; full BASELINE configs are checked on
EVERY row in tests/test_gpu_full_layers.py (every path), plus the V == 1 invariant here.
"""
import math

import numpy as np
import pytest

import oracle
import workloads as W
from tests.gpu_util import oracle_mask, qkv

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

TORCH = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}


def _ulp_half(dtype, ref):
    mant = {"f16": 10, "bf16": 7, "f32": 23}[dtype]
    e = np.floor(np.log2(np.maximum(np.abs(ref), 2.0 ** -14)))
    return 0.5 * 2.0 ** (e - mant)


def run_case(kind, B, H, S, D, dtype, *, causal=False, kv_len=None, layout=None, window=0, n_global=0,
             tile_n=0, fused=True, seed=0, out_f32=True, fuse_ir=False, ir_kernel=False, one_kernel=False,
             two_kernels=False, gs_prologue=False, split_kv=False, concurrent=False, sd=False):
    t, q, k, v = qkv(B, H, S, D, dtype, seed)
    scale = 1 / math.sqrt(D)
    od = torch.float32 if out_f32 else TORCH[dtype]
    kw = dict(scale=scale, causal=causal, tile_n=tile_n, fused=fused, out_dtype=od, fuse_ir=fuse_ir,
              ir_kernel=ir_kernel, one_kernel=one_kernel, two_kernels=two_kernels, gs_prologue=gs_prologue,
              split_kv=split_kv, concurrent=concurrent, sd=sd)
    if kind == "dense":
        o = sr.mha_dense(q, k, v, kv_len=kv_len, **kw)
    elif kind == "block":
        o = sr.mha_blocksparse(q, k, v, layout, **kw)
    else:
        o = sr.mha_sliding_window(q, k, v, window, n_global, **kw)
    torch.cuda.synchronize()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale,
                           oracle_mask(kind, kv_len, causal, layout, window, n_global))
    return o.float().cpu().numpy().astype(np.float64), ref


def assert_close(o, ref, dtype, out_f32=True, what=""):
    err = np.abs(o - ref)
    if dtype == "f32":
        tol = 1e-5
    elif out_f32:
        tol = 1e-2
    else:
        tol = 1e-2 + _ulp_half(dtype, ref)
    bad = err > tol
    assert not bad.any(), f"{what}: {bad.sum()} elements over tolerance, max err {err.max():.3g}"
    assert np.isfinite(o).all()
    return float(err.max())


# ------------------------------------------------------------------------------------ fp32 path

def test_config1_fp32():
    cfg = W.config(1)
    t = W.config_tensors(cfg)
    from tests.gpu_util import to_dev
    q, k, v = (to_dev(x, "f32") for x in (t.q_s, t.k_s, t.v_s))
    o = sr.mha_dense(q, k, v, scale=cfg.scale).cpu().numpy()
    ref = oracle.attention(t.q64, t.k64, t.v64, cfg.scale)
    assert np.abs(o - ref).max() <= 1e-5


def test_p3_closed_form_fp32_with_intermediates():
    """Pin P3 at the C1 shape through the GPU: O, and m', d', r' read back from the workspace."""
    S, D, T = 128, 64, 64
    q = torch.zeros(1, 1, S, D)
    k = torch.zeros(1, 1, S, D)
    for i in range(4):
        q[0, 0, i, i] = math.log(3.0)
        k[0, 0, i, i] = 1.0
    q, k = q.cuda(), k.cuda()
    v = k.clone()
    mask = sr.dense_mask(None)
    info = sr.workspace_info(mask, 1, 1, S, D, sr.SR_F32, tile_n=T)
    ws = torch.zeros(info["total_bytes"], dtype=torch.uint8, device="cuda")
    o = sr.call(mask, q, k, v, scale=1.0, tile_n=T, workspace=ws).cpu().numpy()[0, 0]
    want = np.zeros((S, D))
    for i in range(S):
        for c in range(4):
            want[i, c] = (3.0 if c == i else 1.0) / 130 if i < 4 else 1 / 128
    np.testing.assert_allclose(o, want, atol=1e-7)
    n = info["n_slots"] * 128
    mp = ws[info["off_mprime"]:].view(torch.float32)[:n].cpu().numpy().reshape(-1, 128)
    dp = ws[info["off_dprime"]:].view(torch.float32)[:n].cpu().numpy().reshape(-1, 128)
    rp = ws[info["off_rprime"]:].view(torch.float32)[:n].cpu().numpy().reshape(-1, 128)
    # slots of item (head 0, row-block 0): tiles kt = 0, 1
    np.testing.assert_allclose(mp[:2, 0], [math.log(3.0), 0.0], atol=1e-6)
    np.testing.assert_allclose(dp[:2, 0], [22.0, 64.0], rtol=1e-6)
    np.testing.assert_allclose(rp[:2, 0], [3 / 130, 1 / 130], rtol=1e-6)


@pytest.mark.parametrize("kind", ["dense", "causal", "kv", "block", "window"])
def test_fp32_masks(kind):
    B, H, S, D = 2, 2, 256, 64
    kw = {}
    mk = "dense"
    if kind == "causal":
        kw = dict(causal=True)
    elif kind == "kv":
        kw = dict(kv_len=[200, 3])
    elif kind == "block":
        mk, kw = "block", dict(layout=W.random_layout(H, S // 64, 64, 0.4, seed=4))
    elif kind == "window":
        mk, kw = "window", dict(window=100, n_global=5, causal=False)
    o, ref = run_case(mk, B, H, S, D, "f32", **kw)
    assert_close(o, ref, "f32", what=kind)


@pytest.mark.parametrize("B,H,D,tpr", [(2, 8, 64, 4), (1, 8, 128, 8), (1, 4, 64, 16), (1, 2, 128, 32)],
                         ids=["tpr4", "tpr8", "tpr16", "tpr32"])
def test_fp32_threads_per_row(B, H, D, tpr):
    """The fp32 SIMT kernels at each threads-per-row width the host picks from the item count
    (k_simt_f32.cu: the fewest of 4 / 8 / 16 giving >= 2 CTAs per SM on 148 SMs, else 32), with
    S % 128 == 64, causal and a padded batch entry; every element against the oracle at 1e-5."""
    S = 576  # 4.5 row-blocks
    items = B * H * -(-S // 128)
    assert (items >= 74) == (tpr == 4) and (37 <= items < 74) == (tpr == 8) and (19 <= items < 37) == (tpr == 16)
    for kw in (dict(causal=True), dict(kv_len=[S, 333][:B])):
        o, ref = run_case("dense", B, H, S, D, "f32", **kw)
        assert_close(o, ref, "f32", what=f"tpr {tpr} {kw}")


# ------------------------------------------------------------------------------------ tensor cores

DENSE_CASES = [
    # (dtype, D, T, S, causal, kv_len)
    ("f16", 64, 128, 128, False, None),
    ("f16", 64, 128, 384, False, None),
    ("bf16", 64, 128, 256, False, None),
    ("f16", 128, 128, 256, False, None),
    ("bf16", 128, 128, 384, True, None),
    ("f16", 64, 64, 256, True, None),
    ("bf16", 128, 64, 256, True, None),
    ("f16", 64, 128, 512, False, [512, 511, 384, 300, 257, 128, 65, 1]),
    ("f16", 64, 64, 384, True, [384, 100, 1]),
    # T = 0: the library default (the one-launch kernel; fp16 D = 64 with accumulator-side GS)
    ("f16", 64, 0, 128, False, None),
    ("f16", 64, 0, 640, False, None),
    ("f16", 128, 0, 256, False, None),
    ("bf16", 64, 0, 512, False, [512, 511, 384, 300, 257, 128, 65, 1]),
    ("f16", 64, 0, 512, True, [512, 17, 0, 129]),
]


@pytest.mark.parametrize("case", DENSE_CASES, ids=lambda c: f"{c[0]}-D{c[1]}-T{c[2]}-S{c[3]}-c{int(c[4])}-kv{c[5] is not None}")
@pytest.mark.parametrize("fused", [True, False], ids=["recomposed", "unfused"])
def test_dense_tc(case, fused):
    dtype, D, T, S, causal, kv = case
    B = len(kv) if kv else 2
    o, ref = run_case("dense", B, 3, S, D, dtype, causal=causal, kv_len=kv, tile_n=T, fused=fused)
    assert_close(o, ref, dtype, what=str(case))


@pytest.mark.parametrize("dtype", ["f16", "bf16"])
def test_dense_tc_stored_dtype(dtype):
    o, ref = run_case("dense", 2, 2, 256, 128, dtype, causal=True, out_f32=False)
    assert_close(o, ref, dtype, out_f32=False)


@pytest.mark.parametrize("fused", [True, False], ids=["recomposed", "unfused"])
@pytest.mark.parametrize("density,causal,lh", [(0.3, False, 3), (0.6, True, 3), (0.25, False, 1)])
def test_blocksparse_tc(fused, density, causal, lh):
    S, H = 512, 3
    lay = W.random_layout(lh, S // 64, 64, density, seed=int(density * 100) + lh)
    o, ref = run_case("block", 2, H, S, 64, "f16", causal=causal, layout=lay, fused=fused)
    assert_close(o, ref, "f16")


def test_blocksparse_bigbird_small():
    lay = W.bigbird_layout(2, 1024, 64)
    o, ref = run_case("block", 1, 2, 1024, 64, "f16", layout=lay)
    assert_close(o, ref, "f16")


def test_blocksparse_empty_rows():
    """A block-row with no blocks outputs 0 (reading R9)."""
    S, nb = 256, 4
    lay = W.csr_from_sets(64, [[{0, 1}, set(), {2}, {0, 3}]])
    o, ref = run_case("block", 1, 1, S, 64, "f16", layout=lay)
    assert np.all(o[0, 0, 64:128] == 0)
    assert_close(o, ref, "f16")


@pytest.mark.parametrize("fused", [True, False], ids=["recomposed", "unfused"])
@pytest.mark.parametrize("window,n_global,causal,T", [(0, 0, False, 64), (2, 1, False, 64), (126, 8, False, 64),
                                                      (128, 0, True, 64), (130, 64, False, 128),
                                                      (254, 8, True, 128), (512, 8, False, 64)])
def test_window_tc(fused, window, n_global, causal, T):
    o, ref = run_case("window", 1, 2, 768, 64, "f16", window=window, n_global=n_global, causal=causal,
                      tile_n=T, fused=fused)
    assert_close(o, ref, "f16")


def test_unfused_softmax_streams_long_rows():
    """The baseline's row softmax keeps row slices in shared memory sized for the mean row; the few
    longer rows (global tokens here: 32 key tiles against a mean of ~5) take its streaming path."""
    for fused in (False, True):
        o, ref = run_case("window", 1, 2, 2048, 64, "f16", window=128, n_global=8, tile_n=64, fused=fused)
        assert_close(o, ref, "f16", what=f"fused={fused}")


def test_all_block_layouts_nb2():
    """Pin P7 on the GPU: every block layout with non-empty rows at nb = 2 (9 layouts), S = 128."""
    import itertools
    opts = [c for r in (1, 2) for c in itertools.combinations(range(2), r)]
    for rows in itertools.product(opts, repeat=2):
        lay = W.csr_from_sets(64, [list(rows)])
        o, ref = run_case("block", 1, 1, 128, 64, "f16", layout=lay)
        assert_close(o, ref, "f16", what=str(rows))


def test_kv_len_one_and_zero():
    o, ref = run_case("dense", 3, 2, 256, 64, "f16", kv_len=[1, 0, 129])
    assert np.all(o[1] == 0)
    assert_close(o, ref, "f16")


# ------------------------------------------------------------------------------------ intermediates

def test_intermediates_match_recomposed_oracle():
    """m', d', r' read back from the workspace (SR_IR_KERNEL, the mode that writes d' and r') vs the
    oracle's Eq. (2) decomposition (T = 128)."""
    B, H, S, D, T = 1, 2, 384, 64, 128
    t, q, k, v = qkv(B, H, S, D, "f16", seed=3)
    mask = sr.dense_mask(None)
    info = sr.workspace_info(mask, B, H, S, D, sr.SR_F16, causal=True, tile_n=T)
    ws = torch.zeros(info["total_bytes"], dtype=torch.uint8, device="cuda")
    sr.call(mask, q, k, v, scale=0.125, causal=True, tile_n=T, workspace=ws, ir_kernel=True)
    torch.cuda.synchronize()
    _, mp_ref, dp_ref, rp_ref = oracle.recomposed(t.q64, t.k64, t.v64, 0.125, T, oracle.Mask(causal=True))
    n = info["n_slots"] * 128
    get = lambda key: ws[info[key]:].view(torch.float32)[:n].cpu().numpy().reshape(B * H, -1, 128)
    mp, dp, rp = get("off_mprime"), get("off_dprime"), get("off_rprime")
    # causal with T = M = 128: row-block rb owns tiles kt = 0..rb -> slots rb*(rb+1)/2 + kt
    for g in range(B * H):
        for rb in range(S // 128):
            for kt in range(rb + 1):
                s = rb * (rb + 1) // 2 + kt
                rows = slice(rb * 128, rb * 128 + 128)
                np.testing.assert_allclose(mp[g, s], mp_ref[g, kt, rows], atol=2e-5)
                np.testing.assert_allclose(dp[g, s], dp_ref[g, kt, rows], rtol=2e-3)
                np.testing.assert_allclose(rp[g, s], rp_ref[g, kt, rows], rtol=2e-3, atol=1e-7)


@pytest.mark.parametrize("T", [64, 128])
def test_row_statistics_ir_in_gemm1(T):
    """Default mode (IR in GEMM1): the per-row partial (m, d) GEMM1's two IR warps write vs the oracle's Eq. (2) values:
    m = max_k m'_k, and 1/d = max_k r'_k (r'_k = e^{m'_k - m}/d is 1/d on the tile holding the max)."""
    B, H, S, D = 2, 2, 384, 64
    t, q, k, v = qkv(B, H, S, D, "f16", seed=4)
    kv = [384, 200]
    mask = sr.dense_mask(kv)
    info = sr.workspace_info(mask, B, H, S, D, sr.SR_F16, causal=True, tile_n=T)
    ws = torch.zeros(info["total_bytes"], dtype=torch.uint8, device="cuda")
    o = sr.call(mask, q, k, v, scale=0.125, causal=True, tile_n=T, workspace=ws, out_dtype=torch.float32)
    torch.cuda.synchronize()
    om = oracle.Mask(causal=True, kv_len=kv)
    o_ref, mp_ref, dp_ref, rp_ref = oracle.recomposed(t.q64, t.k64, t.v64, 0.125, T, om)
    assert_close(o.double().cpu().numpy(), o_ref, "f16", what="ir_in_gemm1 output")
    n = B * H * S
    rs = ws[info["off_rowstat"]:].view(torch.float32)[:4 * n].cpu().numpy().reshape(4, B * H, S).astype(np.float64)
    with np.errstate(invalid="ignore"):
        m_ref = mp_ref.max(axis=1)  # [BH, S] over the row's sub-vectors
        invd_ref = rp_ref.max(axis=1)
        # the two IR warps' partials (m_a, d_a), (m_b, d_b) of each row: their maximum is the row's m,
        # and d_a e^{m_a - m} + d_b e^{m_b - m} its d
        m = np.maximum(rs[0], rs[2])
        d = rs[1] * np.exp(np.where(rs[0] == -np.inf, -np.inf, rs[0] - m)) + \
            rs[3] * np.exp(np.where(rs[2] == -np.inf, -np.inf, rs[2] - m))
    np.testing.assert_allclose(m, m_ref, atol=2e-5)
    np.testing.assert_allclose(1.0 / d, invd_ref, rtol=2e-3)


def test_T64_equals_T128():
    """Pin P5 on the GPU: sub-vector width 64 and 128 give the same context within tolerance."""
    o64, ref = run_case("dense", 2, 2, 512, 64, "f16", causal=True, tile_n=64)
    o128, _ = run_case("dense", 2, 2, 512, 64, "f16", causal=True, tile_n=128)
    assert np.abs(o64 - o128).max() < 2e-3
    assert_close(o64, ref, "f16")


# ------------------------------------------------------------------------------------ full configs

def _config_call(cfg, t, fused=True, out_f32=True):
    from tests.gpu_util import to_dev
    q, k, v = (to_dev(x, cfg.dtype) for x in (t.q_s, t.k_s, t.v_s))
    od = torch.float32 if out_f32 else None
    if cfg.kind == "dense":
        o = sr.mha_dense(q, k, v, scale=cfg.scale, kv_len=cfg.kv_len, causal=cfg.causal, out_dtype=od, fused=fused)
        m = oracle.Mask(kv_len=cfg.kv_len, causal=cfg.causal)
    elif cfg.kind == "blocksparse":
        lay = W.config_layout(cfg)
        o = sr.mha_blocksparse(q, k, v, lay, scale=cfg.scale, out_dtype=od, fused=fused)
        m = oracle.Mask(kind="block", layout=lay)
    else:
        o = sr.mha_sliding_window(q, k, v, cfg.window, cfg.n_global, scale=cfg.scale, out_dtype=od, fused=fused)
        m = oracle.Mask(kind="window", window=cfg.window, n_global=cfg.n_global)
    torch.cuda.synchronize()
    return o, m


@pytest.mark.parametrize("idx", [2, 3, 4, 5])
def test_full_config_rows_sum_to_one(idx):
    """Pin P4 at full size: with V == 1 every output element equals 1 (all rows keep >= 1 key)."""
    cfg = W.config(idx)
    t = W.config_tensors(cfg)
    t.v_s = np.ones_like(t.v_s) if cfg.dtype != "bf16" else np.full_like(t.v_s, 0x3F80)
    o, _ = _config_call(cfg, t, out_f32=True)
    err = (o - 1).abs().max().item()
    # Bound from the arithmetic: sum_j Y_j with Y = round_dtype(round_f16(X') * r'): each Y_j carries
    # relative error <= 2^-11 (fp16 X') + half an ulp of the MMA operand dtype (2^-11 f16, 2^-9 bf16);
    # a dominant element can carry it whole.  Plus fp32 accumulation noise.
    bound = 2.0 ** -11 + (2.0 ** -9 if cfg.dtype == "bf16" else 2.0 ** -11) + 1e-4
    assert err <= bound, (err, bound)


def test_abi_errors_on_gpu():
    q = torch.zeros(1, 1, 128, 64, dtype=torch.float16, device="cuda")
    with pytest.raises(sr.SrError) as e:
        sr.mha_dense(q, q, q, out=q)
    assert e.value.status == sr.SR_ERR_INVALID
    q2 = torch.zeros(1, 1, 100, 64, dtype=torch.float16, device="cuda")
    with pytest.raises(sr.SrError) as e:
        sr.mha_dense(q2, q2, q2)
    assert e.value.status == sr.SR_ERR_UNSUPPORTED


@pytest.mark.parametrize("idx,T", [(3, 64), (5, 64), (4, 64)])
def test_gemm2_bitwise_deterministic(idx, T):
    """Regression: an early smem-stage release in GS+GEMM2 corrupted 16-lane groups of rows
    intermittently (30/30 runs at C3 with T=64).  The same inputs must give bitwise equal outputs."""
    from tests.gpu_util import to_dev
    cfg = W.config(idx)
    t = W.config_tensors(cfg)
    mask = (sr.window_mask(cfg.window, cfg.n_global) if cfg.kind == "window" else
            sr.block_mask(W.config_layout(cfg)) if cfg.kind == "blocksparse" else sr.dense_mask(cfg.kv_len))
    q, k, v = (to_dev(x, cfg.dtype) for x in (t.q_s, t.k_s, t.v_s))
    run = lambda: sr.call(mask, q, k, v, scale=cfg.scale, causal=cfg.causal, tile_n=T).clone()
    base = run()
    for _ in range(8):
        assert torch.equal(run(), base)


# ------------------------------------------------------------------------------------ fused-IR variant

FUSED_IR_CASES = [
    ("dense", dict(B=8, H=2, S=512, D=64, dtype="f16", kv_len=[512, 511, 384, 300, 257, 128, 65, 1])),
    ("dense", dict(B=2, H=2, S=384, D=128, dtype="bf16", causal=True)),
    ("dense", dict(B=2, H=2, S=256, D=64, dtype="f16", causal=True, tile_n=64)),
    ("dense", dict(B=3, H=2, S=256, D=64, dtype="f16", kv_len=[1, 0, 129])),
    ("block", dict(B=2, H=3, S=512, D=64, dtype="f16", layout="rand")),
    ("window", dict(B=1, H=2, S=768, D=64, dtype="f16", window=254, n_global=8, causal=True)),
]


VARIANTS = ["fuse_ir", "ir_kernel", "one_kernel", "two_kernels", "gs_prologue", "concurrent"]


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("kind,kw", FUSED_IR_CASES, ids=lambda x: str(x)[:40] if isinstance(x, dict) else x)
def test_fused_ir_variant(kind, kw, variant):
    """The other IR placements against the oracle, same tolerance: SR_FUSE_IR (IR folded into
    GEMM2), SR_IR_KERNEL (the paper's standalone IR kernel writing r'),
    SR_ONE_KERNEL (GEMM1 and GEMM2 phases of each CTA in one launch, the 16-bit default),
    SR_TWO_KERNELS (the same chain as two launches) and SR_CONCURRENT (GEMM1 and GEMM2 concurrently
    in one CTA, item hand-over through mbarriers)."""
    kw = dict(kw)
    if kw.get("layout") == "rand":
        kw["layout"] = W.random_layout(kw["H"], kw["S"] // 64, 64, 0.35, seed=8)
    B, H, S, D, dtype = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    o, ref = run_case(kind, B, H, S, D, dtype, **{variant: True}, **kw)
    if kw.get("kv_len") and 0 in kw["kv_len"]:
        assert np.all(o[list(kw["kv_len"]).index(0)] == 0)
    assert_close(o, ref, dtype, what=f"{variant} {kind}")


CONC_CASES = [
    # empty row-blocks (no tile: both item-end notices, nothing to merge) between full ones
    ("block", dict(B=1, H=2, S=512, D=128, dtype="bf16",
                   layout=W.csr_from_sets(64, [[{0, 1}, set(), set(), set(), {2}, {0, 3}, set(), {7}]] * 2))),
    ("block", dict(B=2, H=1, S=512, D=64, dtype="f16",
                   layout=W.csr_from_sets(64, [[set(), set(), {2}, {0, 3}, set(), set(), {1, 5, 6}, set()]]))),
    ("dense", dict(B=3, H=2, S=384, D=128, dtype="f16", kv_len=[0, 200, 384])),  # a head with no key
    ("dense", dict(B=1, H=1, S=128, D=128, dtype="bf16")),                        # one row-block
    ("dense", dict(B=8, H=8, S=1024, D=128, dtype="bf16", causal=True)),          # 512 items: rings wrap
    ("window", dict(B=2, H=2, S=1024, D=128, dtype="bf16", window=510, n_global=8, causal=True)),
]


@pytest.mark.parametrize("kind,kw", CONC_CASES, ids=lambda x: str(x)[:40] if isinstance(x, dict) else x)
def test_concurrent_edge_cases(kind, kw):
    """SR_CONCURRENT (k_conc.cu) on the item hand-over's edge cases: empty items (two tile-less
    notices each), single-row-block layers, many items per CTA (the item_done / item_free rings wrap),
    and both D; every element against the oracle."""
    kw = dict(kw)
    B, H, S, D, dtype = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    o, ref = run_case(kind, B, H, S, D, dtype, concurrent=True, **kw)
    assert_close(o, ref, dtype, what=f"concurrent {kind}")


S64_CASES = [
    ("dense", dict(B=2, H=2, S=192, D=64, dtype="f16", kv_len=[192, 70])),
    ("dense", dict(B=1, H=3, S=320, D=128, dtype="bf16", causal=True)),
    ("window", dict(B=1, H=2, S=448, D=64, dtype="f16", window=254, n_global=8)),
    ("window", dict(B=2, H=1, S=320, D=128, dtype="bf16", window=126, n_global=4, causal=True)),
    ("block", dict(B=1, H=2, S=576, D=64, dtype="f16", layout="rand")),
    ("dense", dict(B=1, H=1, S=64, D=64, dtype="f16")),  # a single 64-row half
]
S64_PATHS = ["default", "unfused", "two_kernels", "ir_kernel", "fuse_ir", "sd", "gs_prologue", "split_kv",
             "concurrent"]


@pytest.mark.parametrize("path", S64_PATHS)
@pytest.mark.parametrize("kind,kw", S64_CASES, ids=lambda x: str(x)[:40] if isinstance(x, dict) else x)
def test_s_multiple_of_64(kind, kw, path):
    """S % 128 == 64 (S % 64 == 0): the last row-block's upper half lies beyond the head;
    every path computes every row of every head against the oracle."""
    kw = dict(kw)
    if kw.get("layout") == "rand":
        kw["layout"] = W.random_layout(kw["H"], kw["S"] // 64, 64, 0.35, seed=13)
    B, H, S, D, dtype = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    extra = {} if path == "default" else ({"fused": False} if path == "unfused" else {path: True})
    o, ref = run_case(kind, B, H, S, D, dtype, **extra, **kw)
    assert_close(o, ref, dtype, what=f"{path} {kind} S={S}")


@pytest.mark.parametrize("dtype,D", [("f16", 64), ("bf16", 128), ("f32", 64)])
def test_s_multiple_of_64_writes_stay_inside_out(dtype, D):
    """One head with S % 128 == 64: nothing is written past out's last row (a sentinel after it)."""
    S = 192
    t, q, k, v = qkv(1, 1, S, D, dtype, seed=14)
    od = torch.float32
    big = torch.full((S * D + 128 * D,), float("nan"), dtype=od, device="cuda")
    out = big[:S * D].view(1, 1, S, D)
    sr.mha_dense(q, k, v, scale=1 / math.sqrt(D), causal=True, out=out, out_dtype=od)
    torch.cuda.synchronize()
    assert torch.isnan(big[S * D:]).all(), "wrote past the head's last row"
    ref = oracle.attention(t.q64, t.k64, t.v64, 1 / math.sqrt(D), oracle_mask("dense", None, True, None, 0, 0))
    assert_close(out.double().cpu().numpy(), ref, dtype)


# ------------------------------------------------------------------------------------ SD variant

@pytest.mark.parametrize("kind,kw", FUSED_IR_CASES, ids=lambda x: str(x)[:40] if isinstance(x, dict) else x)
def test_sd_variant(kind, kw):
    """SR_DECOMPOSE (the paper's SD: standalone LS / IR / GS between plain GEMMs, NEXT-1)."""
    kw = dict(kw)
    if kw.get("layout") == "rand":
        kw["layout"] = W.random_layout(kw["H"], kw["S"] // 64, 64, 0.35, seed=8)
    B, H, S, D, dtype = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    t, q, k, v = qkv(B, H, S, D, dtype, 0)
    scale = 1 / math.sqrt(D)
    mk = {"dense": sr.dense_mask(kw.get("kv_len")), "block": sr.block_mask(kw["layout"]) if "layout" in kw else None,
          "window": sr.window_mask(kw.get("window", 0), kw.get("n_global", 0))}[kind]
    o = sr.call(mk, q, k, v, scale=scale, causal=kw.get("causal", False), tile_n=kw.get("tile_n", 0),
                out_dtype=torch.float32, sd=True)
    torch.cuda.synchronize()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale,
                           oracle_mask(kind, kw.get("kv_len"), kw.get("causal", False), kw.get("layout"),
                                       kw.get("window", 0), kw.get("n_global", 0)))
    assert_close(o.double().cpu().numpy(), ref, dtype, what=f"SD {kind}")


LONG_CASES = [
    # long sequences past every BASELINE config (several thousand key tiles per head): the default
    # path's schedules, workspace offsets (> 2^31 bytes of X' slots addressed in 64-bit) and row
    # statistics at scale; checked on sampled rows (edge rows included) against the oracle
    ("dense", dict(B=1, H=2, S=16384, D=64, dtype="f16", causal=True)),
    ("dense", dict(B=1, H=2, S=8192, D=128, dtype="bf16", kv_len=[8000])),
    ("window", dict(B=1, H=1, S=32768, D=64, dtype="f16", window=512, n_global=8)),
    ("dense", dict(B=1, H=2, S=32768, D=64, dtype="f16")),  # X' = 4 GiB
    # 2048 row-blocks: more IR CTAs than one wave, so the IR kernel takes its 6-tiles-per-warp
    # classes (rows of up to 64 tiles: staged and folded)
    ("dense", dict(B=2, H=16, S=8192, D=64, dtype="f16", causal=True)),
]


@pytest.mark.parametrize("path", ["default", "ir_kernel"])
@pytest.mark.parametrize("kind,kw", LONG_CASES, ids=lambda x: str(x)[:60] if isinstance(x, dict) else x)
def test_long_sequence_sampled_rows(kind, kw, path):
    """ir_kernel: the paper's standalone IR kernel on rows longer than its shared-memory stage
    (S = 16384 causal: up to 128 key tiles per row, the stage holds 64; the rest fold from global
    memory; the window case: 256-tile global rows beside window rows that see no key in a warp's
    staged tiles)."""
    if path == "ir_kernel" and kind == "dense" and kw["S"] > 16384:
        pytest.skip("X' = 4 GiB; the other cases cover the staged and folded IR paths")
    extra = {"ir_kernel": True} if path == "ir_kernel" else {}
    kw = dict(kw)
    B, H, S, D, dtype = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    t, q, k, v = qkv(B, H, S, D, dtype, seed=S)
    scale = 1 / math.sqrt(D)
    if kind == "dense":
        o = sr.mha_dense(q, k, v, scale=scale, kv_len=kw.get("kv_len"), causal=kw.get("causal", False),
                         out_dtype=torch.float32, **extra)
    else:
        o = sr.mha_sliding_window(q, k, v, kw["window"], kw["n_global"], scale=scale, out_dtype=torch.float32,
                                  **extra)
    torch.cuda.synchronize()
    m = oracle_mask(kind, kw.get("kv_len"), kw.get("causal", False), None, kw.get("window", 0), kw.get("n_global", 0))
    rng = np.random.Generator(np.random.PCG64(S + D))
    edge = [0, 1, 63, 64, 127, 128, 4095, 4096, S // 2, S - 129, S - 128, S - 2, S - 1]
    rows = sorted(set([g * S + i for g in range(B * H) for i in edge] + rng.integers(0, B * H * S, 48).tolist()))
    rows = np.array(rows, dtype=np.int64)
    ref = oracle.attention_rows(t.q64, t.k64, t.v64, scale, rows, m)
    got = o.reshape(-1, D)[torch.from_numpy(rows).cuda()].double().cpu().numpy()
    assert_close(got, ref, dtype, what=f"{kind} S={S}")
    assert torch.isfinite(o).all()


# ------------------------------------------------------------------------------------ SR_SPLIT_KV

SPLIT_CASES = [
    # few heads, long rows: the split plan cuts rows into chunks of >= 4 key tiles
    ("dense", dict(B=1, H=2, S=2048, D=128, dtype="bf16", causal=True)),
    ("dense", dict(B=4, H=1, S=1024, D=64, dtype="f16", kv_len=[1024, 1000, 700, 1], causal=True)),
    ("dense", dict(B=1, H=3, S=1024, D=64, dtype="f16")),
    ("window", dict(B=1, H=2, S=4096, D=64, dtype="f16", window=512, n_global=8)),
    ("block", dict(B=1, H=2, S=2048, D=64, dtype="f16", layout="bigbird")),
]


@pytest.mark.parametrize("stored", [False, True], ids=["fp32-context", "stored"])
@pytest.mark.parametrize("kind,kw", SPLIT_CASES, ids=lambda x: str(x)[:50] if isinstance(x, dict) else x)
def test_split_kv(kind, kw, stored):
    """SR_SPLIT_KV (include/sr_mha.h): chunked GEMM1 + LS, IR over whole rows, chunked GS + GEMM2
    writing partial contexts, combine -- every element against the oracle."""
    kw = dict(kw)
    if kw.get("layout") == "bigbird":
        kw["layout"] = W.bigbird_layout(kw["H"], kw["S"], 64)
    B, H, S, D, dtype = (kw.pop(x) for x in ("B", "H", "S", "D", "dtype"))
    o, ref = run_case(kind, B, H, S, D, dtype, split_kv=True, out_f32=not stored, **kw)
    assert_close(o, ref, dtype, out_f32=not stored, what=f"split {kind}")


def test_split_kv_c3_shard():
    """One GPU's share of C3 head-sharded over 8 GPUs (8 causal heads), the case SR_SPLIT_KV is for."""
    from paper_conf_iiswc_choilkha22_b200 import shard as SH
    cfg = W.config(3)
    sh = SH.make_shard(0, 8, cfg.B, cfg.H, cfg.S, T=64, causal=True)
    t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=cfg.idx)
    from tests.gpu_util import to_dev
    q, k, v = (SH.shard_view(to_dev(x, cfg.dtype), sh).contiguous() for x in (t.q_s, t.k_s, t.v_s))
    o = sr.mha_dense(q, k, v, scale=cfg.scale, causal=True, out_dtype=torch.float32, split_kv=True)
    torch.cuda.synchronize()
    q64, k64, v64 = (SH.shard_view(torch.from_numpy(x), sh).numpy() for x in (t.q64, t.k64, t.v64))
    ref = oracle.attention(q64, k64, v64, cfg.scale, oracle.Mask(causal=True))
    assert_close(o.double().cpu().numpy(), ref, cfg.dtype, what="C3 shard split")


@pytest.mark.parametrize("idx", [4, 5])
def test_auto_split_on_global_row_shards(idx):
    """The default call chooses SR_SPLIT_KV by itself when a few long rows dominate the one-launch
    schedule -- one GPU's share of an 8-way head-sharded BigBird / Longformer layer (global rows hold
    every key tile): every element against the oracle, and bitwise equal to the explicit split."""
    from paper_conf_iiswc_choilkha22_b200 import shard as SH
    from tests.gpu_util import to_dev
    cfg = W.config(idx)
    lay = W.config_layout(cfg)
    sh = SH.make_shard(0, 8, cfg.B, cfg.H, cfg.S, layout=lay, T=64)
    t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=cfg.idx)
    q, k, v = (SH.shard_view(to_dev(x, cfg.dtype), sh).contiguous() for x in (t.q_s, t.k_s, t.v_s))
    if cfg.kind == "blocksparse":
        mask, om = sr.block_mask(sh.layout), oracle.Mask(kind="block", layout=sh.layout)
    else:
        mask = sr.window_mask(cfg.window, cfg.n_global)
        om = oracle.Mask(kind="window", window=cfg.window, n_global=cfg.n_global)
    n0 = sr.launch_count()
    o = sr.call(mask, q, k, v, scale=cfg.scale, out_dtype=torch.float32)
    torch.cuda.synchronize()
    assert sr.launch_count() - n0 >= 4, "expected the split path (upload, GEMM1, IR, GEMM2, combine)"
    o2 = sr.call(mask, q, k, v, scale=cfg.scale, out_dtype=torch.float32, split_kv=True)
    torch.cuda.synchronize()
    assert torch.equal(o, o2)
    q64, k64, v64 = (SH.shard_view(torch.from_numpy(x), sh).numpy() for x in (t.q64, t.k64, t.v64))
    ref = oracle.attention(q64, k64, v64, cfg.scale, om)
    assert_close(o.double().cpu().numpy(), ref, cfg.dtype, what=f"C{idx} shard auto split")
