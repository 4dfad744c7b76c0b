"""Pins of the fp64 oracle against things other than itself (task rule ③).

Every test here is CPU-only. A plausible mistake anywhere in the oracle -- a dropped term, a wrong
sign, a transposed operand, an off-by-one in a mask, a wrong reconstruction factor -- fails at
least one of them:
  P1/P2  hand-worked 4x4 fixtures (tests/golden/*.txt): exact values of O, m', d', r'
  P3     closed forms at GPU shapes (S=128, D=64, T=64), dense and causal
  P4     V == 1  =>  O == 1 (every kept softmax row sums to 1)
  P5     Eq. (2) recomposition == Eq. (1) for several T ("mathematically identical")
  P6     shift / permutation invariance, linearity in V, kv_len = 1 => O_i = V_0
  P7     brute force: all 2^16 element masks at S=4; all block layouts at nb=2; window params
  P8     library routines: numpy fp64 (independent mask construction) and torch SDPA (fp64)
  layout counts: BigBird 622 blocks/head, Longformer 2,096,824 kept elements/head (closed form)
"""
import itertools
import math

import numpy as np
import pytest

import oracle
import workloads as W
from oracle import oracle_np
from tests.golden_io import load

LN3 = math.log(3.0)


def _eye_problem(S, D, n, c):
    q = np.zeros((1, 1, S, D))
    k = np.zeros((1, 1, S, D))
    for i in range(n):
        q[0, 0, i, i] = c
        k[0, 0, i, i] = 1.0
    return q, k, k.copy()


def _golden_case(name):
    g = load(name)
    S = int(g["S"])
    q, k, v = _eye_problem(S, S, S, g["q_diag"])
    mask = oracle.Mask(kind="none", causal=bool(g.get("causal", 0)),
                       kv_len=[int(g["kv_len"])] if "kv_len" in g else None)
    return g, q, k, v, mask


@pytest.mark.parametrize("name", ["p1_4x4_dense.txt", "p2_4x4_causal.txt", "p2_4x4_kvlen3.txt"])
def test_p1_p2_golden(name):
    g, q, k, v, mask = _golden_case(name)
    want = np.array(g["O"])
    o = oracle.attention(q, k, v, g["scale"], mask)[0, 0]
    np.testing.assert_allclose(o, want, rtol=0, atol=1e-15)
    T = int(g.get("T", 2))
    o2, mp, dp, rp = oracle.recomposed(q, k, v, g["scale"], T, mask)
    np.testing.assert_allclose(o2[0, 0], want, rtol=0, atol=1e-15)
    if "row" in g:
        r = int(g["row"])
        np.testing.assert_allclose(mp[0, :, r], g["mprime"], rtol=0, atol=1e-15)
        np.testing.assert_allclose(dp[0, :, r], g["dprime"], rtol=0, atol=1e-15)
        np.testing.assert_allclose(rp[0, :, r], g["rprime"], rtol=0, atol=1e-15)


def p3_expected(S, D, n, a, causal):
    """Closed form for the identity embedding: q_i = c e_i, k_i = v_i = e_i (i < n), zero rows
    elsewhere, a = e^{c*scale}. Row i < n: scores c*scale at j = i, 0 at the other kept j."""
    O = np.zeros((S, D))
    for i in range(S):
        kept = (i + 1) if causal else S
        if i < n:
            den = a + (kept - 1)
            for c in range(min(n, kept)):
                O[i, c] = (a if c == i else 1.0) / den
        else:
            for c in range(min(n, kept)):
                O[i, c] = 1.0 / kept
    return O


@pytest.mark.parametrize("causal", [False, True])
def test_p3_closed_form_gpu_shape(causal):
    S, D, n, T = 128, 64, 4, 64
    q, k, v = _eye_problem(S, D, n, LN3)
    mask = oracle.Mask(causal=causal)
    want = p3_expected(S, D, n, 3.0, causal)
    if not causal:  # the SURVEY's printed forms
        assert abs(want[0, 0] - 3 / 130) < 1e-18 and abs(want[0, 1] - 1 / 130) < 1e-18
        assert abs(want[5, 2] - 1 / 128) < 1e-18
    o = oracle.attention(q, k, v, 1.0, mask)[0, 0]
    np.testing.assert_allclose(o, want, rtol=0, atol=5e-16)
    o2, mp, dp, rp = oracle.recomposed(q, k, v, 1.0, T, mask)
    np.testing.assert_allclose(o2[0, 0], want, rtol=0, atol=5e-16)
    if not causal:
        np.testing.assert_allclose(mp[0, :, 0], [LN3, 0.0], atol=1e-15)
        np.testing.assert_allclose(dp[0, :, 0], [22.0, 64.0], atol=1e-13)
        np.testing.assert_allclose(rp[0, :, 0], [3 / 130, 1 / 130], atol=1e-16)


def test_p3_dtype_variant_scale():
    """c = 1.0 (exact in f16/bf16) with scale 1/sqrt(D): a = e^{1/8} replaces 3."""
    S, D, n = 128, 64, 4
    q, k, v = _eye_problem(S, D, n, 1.0)
    scale = 1 / math.sqrt(D)
    o = oracle.attention(q, k, v, scale)[0, 0]
    np.testing.assert_allclose(o, p3_expected(S, D, n, math.exp(scale), False), atol=1e-16)


def _rand(B, H, S, D, seed):
    t = W.make_qkv(B, H, S, D, "f32", seed_base=seed)
    return t.q64, t.k64, t.v64


def _masks(B, H, S):
    lay = W.random_layout(H, S // 16, 16, 0.3, seed=7)
    return [
        ("none", oracle.Mask()),
        ("causal", oracle.Mask(causal=True)),
        ("kvlen", oracle.Mask(kv_len=np.arange(B) * 7 % S + 1)),
        ("kvlen_causal", oracle.Mask(kv_len=np.arange(B) * 5 % S + 3, causal=True)),
        ("block", oracle.Mask(kind="block", layout=lay)),
        ("block_causal", oracle.Mask(kind="block", layout=lay, causal=True)),
        ("window", oracle.Mask(kind="window", window=10, n_global=2)),
        ("window_causal", oracle.Mask(kind="window", window=6, n_global=1, causal=True)),
    ]


def test_p4_rows_sum_to_one():
    B, H, S, D = 2, 3, 64, 8
    q, k, _ = _rand(B, H, S, D, 11)
    v = np.ones((B, H, S, D))
    lay = W.random_layout(H, S // 16, 16, 0.3, seed=7)
    specs = {"none": {}, "causal": dict(causal=True), "kvlen": dict(kv_len=np.arange(B) * 7 % S + 1),
             "kvlen_causal": dict(kv_len=np.arange(B) * 5 % S + 3, causal=True),
             "block": dict(kind="block", layout=lay), "block_causal": dict(kind="block", layout=lay, causal=True),
             "window": dict(kind="window", window=10, n_global=2),
             "window_causal": dict(kind="window", window=6, n_global=1, causal=True)}
    for name, m in _masks(B, H, S):
        o = oracle.attention(q, k, v, 0.3, m)
        # rows that keep >= 1 element sum to 1; rows that keep none output 0 (reading R9).
        # The kept-row set comes from numpy's independent mask construction.
        for b in range(B):
            for h in range(H):
                live = oracle_np.allowed_matrix(S, b=b, h=h, **specs[name]).any(axis=1)
                want = np.where(live[:, None], 1.0, 0.0)
                np.testing.assert_allclose(o[b, h], np.broadcast_to(want, (S, D)), rtol=0, atol=1e-13,
                                           err_msg=name)


@pytest.mark.parametrize("T", [1, 2, 16, 64, 128, 256, 48])
def test_p5_recomposed_equals_monolithic(T):
    B, H, S, D = 1, 2, 256, 16
    q, k, v = _rand(B, H, S, D, 5)
    for name, m in [("none", oracle.Mask()), ("causal", oracle.Mask(causal=True)),
                    ("window", oracle.Mask(kind="window", window=40, n_global=3)),
                    ("kv", oracle.Mask(kv_len=[77]))]:
        o1 = oracle.attention(q, k, v, 0.25, m)
        o2, mp, dp, rp = oracle.recomposed(q, k, v, 0.25, T, m)
        np.testing.assert_allclose(o2, o1, rtol=0, atol=5e-15, err_msg=f"{name} T={T}")
        # reconstruction factors times local sums add to one per row (IR definition)
        with np.errstate(invalid="ignore"):
            s = (rp * dp).sum(axis=1)
        np.testing.assert_allclose(s, 1.0, atol=1e-13)


def test_p6_invariances():
    B, H, S, D = 1, 2, 96, 12
    q, k, v = _rand(B, H, S, D, 3)
    scale = 0.4
    o = oracle.attention(q, k, v, scale)
    # shift: K + 1 u^T adds q_i.u to every score of row i
    u = np.linspace(-2, 3, D)
    np.testing.assert_allclose(oracle.attention(q, k + u, v, scale), o, atol=1e-13)
    # joint permutation of keys and values (no mask)
    perm = np.random.Generator(np.random.PCG64(1)).permutation(S)
    np.testing.assert_allclose(oracle.attention(q, k[:, :, perm], v[:, :, perm], scale), o, atol=1e-13)
    # linearity in V
    v2 = np.cos(v * 3)
    np.testing.assert_allclose(oracle.attention(q, k, v + v2, scale),
                               o + oracle.attention(q, k, v2, scale), atol=1e-13)
    # kv_len = 1: every row sees key 0 only
    o1 = oracle.attention(q, k, v, scale, oracle.Mask(kv_len=[1]))
    np.testing.assert_allclose(o1, np.broadcast_to(v[:, :, :1, :], o1.shape), rtol=0, atol=0)
    # a row that sees nothing outputs 0 (reading R9)
    o0 = oracle.attention(q, k, v, scale, oracle.Mask(kv_len=[0]))
    assert np.all(o0 == 0)


def test_p7_all_element_masks_S4():
    S, D = 4, 3
    n = 1 << (S * S)
    bits = ((np.arange(n)[:, None] >> np.arange(S * S)[None, :]) & 1).astype(np.uint8)
    elem = bits.reshape(n, S, S)
    rng = np.random.Generator(np.random.PCG64(9))
    q = np.broadcast_to(rng.standard_normal((1, 1, S, D)), (1, n, S, D)).copy()
    k = np.broadcast_to(rng.standard_normal((1, 1, S, D)), (1, n, S, D)).copy()
    v = np.broadcast_to(rng.standard_normal((1, 1, S, D)), (1, n, S, D)).copy()
    m = oracle.Mask(kind="elem", elem=elem)
    o_c = oracle.attention(q, k, v, 0.7, m)
    o_r2, *_ = oracle.recomposed(q, k, v, 0.7, 2, m)
    o_r3, *_ = oracle.recomposed(q, k, v, 0.7, 3, m)
    # numpy, dense-masked, batched over the 2^16 masks
    x = 0.7 * np.einsum("id,jd->ij", q[0, 0], k[0, 0])
    xm = np.where(elem.astype(bool), x[None], -np.inf)
    mx = xm.max(axis=2, keepdims=True)
    e = np.where(elem.astype(bool), np.exp(xm - np.where(np.isfinite(mx), mx, 0)), 0.0)
    d = e.sum(axis=2, keepdims=True)
    p = np.where(d > 0, e / np.where(d > 0, d, 1), 0.0)
    o_np = p @ v[0, 0]
    np.testing.assert_allclose(o_c[0], o_np, atol=1e-14)
    np.testing.assert_allclose(o_r2[0], o_np, atol=1e-14)
    np.testing.assert_allclose(o_r3[0], o_np, atol=1e-14)


def test_p7_all_block_layouts_nb2():
    S, D, blk, nb = 4, 3, 2, 2
    q, k, v = _rand(1, 1, S, D, 21)
    rows_opts = [c for r in range(1, nb + 1) for c in itertools.combinations(range(nb), r)]
    count = 0
    for rows in itertools.product(rows_opts, repeat=nb):
        lay = W.csr_from_sets(blk, [list(rows)])
        m = oracle.Mask(kind="block", layout=lay)
        want = oracle_np.attention(q, k, v, 0.5, kind="block", layout=lay)
        np.testing.assert_allclose(oracle.attention(q, k, v, 0.5, m), want, atol=1e-14)
        for causal in (False, True):
            mc = oracle.Mask(kind="block", layout=lay, causal=causal)
            a_np = oracle_np.allowed_matrix(S, kind="block", layout=lay, causal=causal)
            assert oracle.count_allowed(1, 1, S, mc)[0] == a_np.sum()
        count += 1
    assert count == 9


@pytest.mark.parametrize("window,n_global", list(itertools.product([0, 2, 6, 126, 128, 130, 254], [0, 1, 8, 64])))
def test_p7_window_predicate(window, n_global):
    S = 256
    for causal in (False, True):
        m = oracle.Mask(kind="window", window=window, n_global=n_global, causal=causal)
        a = oracle_np.allowed_matrix(S, kind="window", window=window, n_global=n_global, causal=causal)
        assert oracle.count_allowed(1, 1, S, m)[0] == int(a.sum())


def test_p8_numpy_and_torch_sdpa():
    torch = pytest.importorskip("torch")
    B, H, S, D = 2, 3, 80, 16
    q, k, v = _rand(B, H, S, D, 31)
    scale = 1 / math.sqrt(D)
    lay = W.random_layout(H, S // 16, 16, 0.35, seed=3)
    cases = [dict(kind="none"), dict(kind="none", causal=True), dict(kind="none", kv_len=[80, 17]),
             dict(kind="block", layout=lay), dict(kind="window", window=12, n_global=3),
             dict(kind="window", window=30, n_global=2, causal=True)]
    for c in cases:
        o = oracle.attention(q, k, v, scale, oracle.Mask(**c))
        o_np = oracle_np.attention(q, k, v, scale, **c)
        np.testing.assert_allclose(o, o_np, atol=1e-14, err_msg=str(c))
        am = np.stack([np.stack([oracle_np.allowed_matrix(S, b=b, h=h, **c) for h in range(H)])
                       for b in range(B)])
        ot = torch.nn.functional.scaled_dot_product_attention(
            torch.from_numpy(q), torch.from_numpy(k), torch.from_numpy(v),
            attn_mask=torch.from_numpy(am), scale=scale).numpy()
        np.testing.assert_allclose(o, ot, atol=1e-13, err_msg=str(c))


def test_rows_api_matches_full():
    B, H, S, D = 2, 2, 64, 8
    q, k, v = _rand(B, H, S, D, 2)
    m = oracle.Mask(kind="window", window=16, n_global=2, causal=True)
    o = oracle.attention(q, k, v, 0.3, m).reshape(-1, D)
    rows = np.array([0, 5, 63, 64, 200, 255])
    np.testing.assert_array_equal(oracle.attention_rows(q, k, v, 0.3, rows, m), o[rows])


def test_layout_counts_bigbird():
    cfg = W.config(4)
    lay = W.config_layout(cfg)
    nb = cfg.S // cfg.block
    assert lay.layout_heads == cfg.H
    for h in range(cfg.H):
        assert lay.nnz(h) == 622
        counts = [len(lay.blocks(h, r)) for r in range(nb)]
        assert counts[0] == counts[-1] == nb
        assert counts[1] == counts[-2] == 7
        assert all(c == 8 for c in counts[2:-2])
    # the C predicate agrees with the CSR: 622 blocks of 64x64 kept per head
    m = oracle.Mask(kind="block", layout=lay)
    tot, per = oracle.count_allowed(1, 2, cfg.S, m)
    assert list(per) == [622 * 64 * 64] * 2


def test_layout_counts_longformer_closed_form():
    S, w, g = 4096, 256, 8
    band = S * (2 * w + 1) - w * (w + 1)
    glob_rows = sum(S - (i + w + 1) for i in range(g))
    closed = band + 2 * glob_rows
    assert closed == 2_096_824
    m = oracle.Mask(kind="window", window=512, n_global=8)
    assert oracle.count_allowed(1, 1, S, m)[0] == closed
