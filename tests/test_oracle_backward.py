"""Pins of the backward oracle (oracle/backward.py, §6 Eq. 3) against
things other than itself.  CPU only.

  B1  central finite differences of the FORWARD oracle (the C textbook attention), so the
      gradient formulas are checked against nothing but the forward definition
  B2  literal Eq. (3) Jacobian (dy_i/dx_k = y_i(1-y_i) / -y_i y_k) vs the row form, incl. masked
      entries (y = 0)
  B3  torch.autograd through fp64 scaled_dot_product_attention (library routine), with masks
  B4  invariants: V = const rows => dQ = dK = 0; sum_j dV_j = sum_i dO_i (softmax rows sum to 1);
      sum_k dX_k = 0 per row; fully masked rows give zero gradients and zero output
  B5  the forward half of attention_backward equals the C oracle's O (masks, sparse layouts)
A dropped y_k factor, a sign flip of the sum term, a missing scale, a transposed dX or an
unmasked element fails at least one of them.
"""
import numpy as np
import pytest

import oracle
import workloads as W
from oracle import backward as OB
from oracle import oracle_np


def _rand(shape, seed, s=1.0):
    return s * np.random.Generator(np.random.PCG64(seed)).standard_normal(shape)


def _loss_grad_fd(q, k, v, do, scale, mask, eps=1e-6):
    """dE/dq, dE/dk, dE/dv of E = <dO, O(q, k, v)> by central differences of the C oracle."""
    def E(q_, k_, v_):
        return float((oracle.attention(q_, k_, v_, scale, mask) * do).sum())
    grads = []
    for which in range(3):
        base = [q.copy(), k.copy(), v.copy()]
        g = np.zeros_like(base[which])
        it = np.nditer(g, flags=["multi_index"])
        for _ in it:
            idx = it.multi_index
            p = [x.copy() for x in base]
            m = [x.copy() for x in base]
            p[which][idx] += eps
            m[which][idx] -= eps
            g[idx] = (E(*p) - E(*m)) / (2 * eps)
        grads.append(g)
    return grads


@pytest.mark.parametrize("case", ["dense", "causal", "kvlen", "window"])
def test_b1_finite_differences(case):
    B, H, S, D = 1, 2, 6, 3
    q, k, v, do = (_rand((B, H, S, D), s) for s in (11, 12, 13, 14))
    scale = 0.7
    kw = {"dense": {}, "causal": {"causal": True}, "kvlen": {"kv_len": [4]},
          "window": {"kind": "window", "window": 2, "n_global": 1}}[case]
    cmask = oracle.Mask(kind=kw.get("kind", "none"), kv_len=kw.get("kv_len"), causal=kw.get("causal", False),
                        window=kw.get("window", 0), n_global=kw.get("n_global", 0))
    _, dq, dk, dv = OB.attention_backward(q, k, v, do, scale, **kw)
    fq, fk, fv = _loss_grad_fd(q, k, v, do, scale, cmask)
    for a, b in ((dq, fq), (dk, fk), (dv, fv)):
        assert np.abs(a - b).max() < 1e-7, np.abs(a - b).max()


def test_b2_literal_jacobian():
    rng = np.random.Generator(np.random.PCG64(5))
    for L in (1, 2, 5, 17):
        x = rng.standard_normal((3, L)) * 2
        x[1, : L // 2] = -np.inf  # partially masked row (y = 0 there)
        y = OB.softmax_rows(x)
        dy = rng.standard_normal((3, L))
        rows = OB.softmax_backward_rows(y, dy)
        for r in range(3):
            lit = OB.softmax_backward_eq3(y[r], dy[r])
            assert np.abs(lit - rows[r]).max() < 1e-14
        assert np.all(rows[1, : L // 2] == 0.0)


def test_b3_torch_autograd():
    torch = pytest.importorskip("torch")
    B, H, S, D = 2, 3, 40, 8
    q, k, v, do = (_rand((B, H, S, D), s) for s in (21, 22, 23, 24))
    scale = 1 / np.sqrt(D)
    kv = [29, 40]
    for kw in ({}, {"causal": True}, {"kv_len": kv}, {"kind": "window", "window": 10, "n_global": 3}):
        _, dq, dk, dv = OB.attention_backward(q, k, v, do, scale, **kw)
        allowed = np.stack([oracle_np.allowed_matrix(S, b=b, h=h, **kw) for b in range(B) for h in range(H)])
        tq, tk, tv = (torch.tensor(x, requires_grad=True) for x in (q, k, v))
        am = torch.tensor(allowed.reshape(B, H, S, S))
        o = torch.nn.functional.scaled_dot_product_attention(tq, tk, tv, attn_mask=am, scale=scale)
        o.backward(torch.tensor(do))
        for a, t in ((dq, tq), (dk, tk), (dv, tv)):
            assert np.abs(a - t.grad.numpy()).max() < 1e-12


def test_b4_invariants():
    B, H, S, D = 1, 2, 64, 16
    q, k, do = (_rand((B, H, S, D), s) for s in (31, 32, 34))
    scale = 0.25
    # V = the same vector in every row: O does not depend on the scores => dQ = dK = 0
    v = np.broadcast_to(_rand((1, 1, 1, D), 33), (B, H, S, D)).copy()
    _, dq, dk, dv = OB.attention_backward(q, k, v, do, scale, causal=True)
    assert np.abs(dq).max() < 1e-12 and np.abs(dk).max() < 1e-12
    # sum_j dV_j = sum_i y_ij dO_i summed over j = sum_i dO_i (rows of y sum to 1)
    v = _rand((B, H, S, D), 35)
    _, dq, dk, dv = OB.attention_backward(q, k, v, do, scale, kv_len=[37])
    assert np.abs(dv.sum(axis=2) - do.sum(axis=2)).max() < 1e-11
    # sum_k dX_k = 0  <=>  dQ = scale * dX K is unchanged by adding a constant row to K
    _, dq2, _, _ = OB.attention_backward(q, k + _rand((1, 1, 1, D), 36), v, do, scale, kv_len=[37])
    assert np.abs(dq2 - dq).max() < 1e-11
    # keys past kv_len get no gradient; a fully masked row (kv_len = 0) gives zeros everywhere
    assert np.all(dk[:, :, 37:] == 0) and np.all(dv[:, :, 37:] == 0)
    O, dq, dk, dv = OB.attention_backward(q, k, v, do, scale, kv_len=[0])
    assert not O.any() and not dq.any() and not dk.any() and not dv.any()


def test_b5_forward_matches_c_oracle():
    B, H, S, D = 1, 2, 256, 16
    t = W.make_qkv(B, H, S, D, "f16", seed_base=3)
    lay = W.random_layout(H, S // 64, 64, 0.4, seed=9)
    for kw, cm in (({"kind": "block", "layout": lay, "causal": True}, oracle.Mask("block", layout=lay, causal=True)),
                   ({"kind": "window", "window": 64, "n_global": 5}, oracle.Mask("window", window=64, n_global=5))):
        O, *_ = OB.attention_backward(t.q64, t.k64, t.v64, np.zeros_like(t.q64), 0.25, **kw)
        assert np.abs(O - oracle.attention(t.q64, t.k64, t.v64, 0.25, cm)).max() < 1e-13
