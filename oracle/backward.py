"""fp64 CPU oracle of the attention layer's backward pass -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s CPU legs may import this module;
the CUDA path shares no code with it.

What it computes (§6 "Applying softmax recomposition to training", L247-L253, and the
attention layer of L51-L53), per head, in fp64 on the dtype-rounded inputs:

    x  = scale * Q K^T, masked elements -inf                  (L51-L53: MatMul, divide, mask)
    y  = softmax(x) row-wise (Eq. 1); a row with no kept key has y = 0 (reading R9)
    O  = y V                                                   (L53)
    dY = dO V^T            (dE/dy_ij = sum_d dE/dO_id V_jd: the derivative of O = y V)
    dX = Eq. (3):  dE/dx_k = sum_i dE/dy_i * dy_i/dx_k,  dy_i/dx_k = y_i (1 - y_i) if i = k,
                                                                   -y_i y_k     otherwise
         evaluated per row as  dX_k = y_k (dY_k - sum_i dY_i y_i)   (the same sum: the i = k term
         contributes y_k dY_k and every term carries a factor y_k; `softmax_backward_eq3` below
         writes the Jacobian out literally and the pins check the two agree)
    dV = y^T dO,  dQ = scale * dX K,  dK = scale * dX^T Q      (derivatives of the MatMuls)

Masked elements have y = 0, so their dX is 0 and they contribute nothing -- the paper's point
(L251-L253): the backward needs only y (and dY), never the softmax input x.

Parity status: pinned in ``tests/test_oracle_backward.py`` against central finite differences
of the forward oracle (independent of every formula above), ``torch.autograd`` on fp64
``scaled_dot_product_attention`` (library routine), the literal Jacobian of Eq. 3, and the
invariants V = const => dQ = dK = 0, sum_j dV_j = sum_i dO_i (rows of y sum to 1) and
sum_k dX_k = 0 per row.
"""
from __future__ import annotations

import numpy as np

from .oracle_np import allowed_matrix


def softmax_rows(x: np.ndarray) -> np.ndarray:
    """Eq. (1) per row; -inf entries give 0; an all -inf row gives all zeros (reading R9)."""
    m = x.max(axis=1, keepdims=True)
    live = np.isfinite(m[:, 0])
    e = np.exp(x - np.where(live[:, None], m, 0.0))
    e[~np.isfinite(x)] = 0.0
    d = e.sum(axis=1, keepdims=True)
    return np.where(live[:, None], e / np.where(d > 0, d, 1.0), 0.0)


def softmax_backward_eq3(y_row: np.ndarray, dy_row: np.ndarray) -> np.ndarray:
    """Eq. (3) written out literally for ONE row: the L x L Jacobian dy_i/dx_k, then
    dE/dx_k = sum_i dE/dy_i * dy_i/dx_k.  O(L^2): small rows only (pins)."""
    L = y_row.shape[0]
    J = np.empty((L, L))
    for i in range(L):
        for k in range(L):
            J[i, k] = y_row[i] * (1.0 - y_row[i]) if i == k else -y_row[i] * y_row[k]
    return dy_row @ J


def softmax_backward_rows(y: np.ndarray, dy: np.ndarray) -> np.ndarray:
    """Eq. (3) for every row at once: dX_k = y_k (dY_k - sum_i dY_i y_i)."""
    return y * (dy - (dy * y).sum(axis=1, keepdims=True))


def attention_backward(q, k, v, do, scale, heads=None, **mask):
    """q, k, v, do: fp64 [B, H, S, D].  Returns (O, dQ, dK, dV), fp64 [B, H, S, D] (only the flat
    heads g = b*H + h listed in ``heads`` are computed if given; the others stay 0).
    ``mask``: the keyword arguments of oracle_np.allowed_matrix (kind, kv_len, causal, layout,
    window, n_global, elem)."""
    B, H, S, D = q.shape
    O, dQ, dK, dV = (np.zeros((B, H, S, D)) for _ in range(4))
    elem = mask.pop("elem", None)
    for g in (range(B * H) if heads is None else heads):
        b, h = divmod(int(g), H)
        a = allowed_matrix(S, b=b, h=h, elem=None if elem is None else elem[g], **mask)
        x = np.where(a, scale * (q[b, h] @ k[b, h].T), -np.inf)
        y = softmax_rows(x)
        O[b, h] = y @ v[b, h]
        dy = do[b, h] @ v[b, h].T
        dx = softmax_backward_rows(y, dy)
        dV[b, h] = y.T @ do[b, h]
        dQ[b, h] = scale * (dx @ k[b, h])
        dK[b, h] = scale * (dx.T @ q[b, h])
    return O, dQ, dK, dV
