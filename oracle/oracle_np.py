"""numpy fp64 cross-check of the C oracle -- TEST INFRASTRUCTURE ONLY.

A second, independently written statement of the same definition (Eq. 1):
the mask is materialised as a dense boolean matrix by numpy broadcasting (not by the C
predicate), scores by a library matmul, softmax by vectorised max/exp/sum. It exists so the C
oracle can be pinned against something other than itself (SURVEY §8(c) pin P8). Only tests/ may
import it.
"""
from __future__ import annotations

import numpy as np


def allowed_matrix(S, *, b=0, h=0, kind="none", kv_len=None, causal=False, layout=None,
                   window=0, n_global=0, elem=None):
    """Dense [S, S] boolean mask for head (b, h); True = element kept."""
    i = np.arange(S)[:, None]
    j = np.arange(S)[None, :]
    a = np.ones((S, S), dtype=bool)
    if kind == "block":
        nb = S // layout.block
        lh = 0 if layout.layout_heads == 1 else h
        blk = np.zeros((nb, nb), dtype=bool)
        for r in range(nb):
            blk[r, layout.blocks(lh, r)] = True
        a = np.kron(blk, np.ones((layout.block, layout.block), dtype=bool)).astype(bool)
    elif kind == "window":
        a = (np.abs(i - j) <= window // 2) | (i < n_global) | (j < n_global)
    elif kind == "elem":
        a = elem.astype(bool).copy()
    if kv_len is not None:
        a &= j < int(kv_len[b])
    if causal:
        a &= j <= i
    return a


def attention(q, k, v, scale, **mask):
    """q, k, v: fp64 [B, H, S, D]. Returns fp64 [B, H, S, D]."""
    B, H, S, D = q.shape
    out = np.zeros_like(q)
    elem = mask.pop("elem", None)
    for b in range(B):
        for h in range(H):
            e = None if elem is None else elem[b * H + h]
            a = allowed_matrix(S, b=b, h=h, elem=e, **mask)
            x = scale * (q[b, h] @ k[b, h].T)
            x = np.where(a, x, -np.inf)
            m = x.max(axis=1, keepdims=True)
            live = np.isfinite(m[:, 0])
            e_ = np.where(a, np.exp(x - np.where(np.isfinite(m), m, 0.0)), 0.0)
            d = e_.sum(axis=1, keepdims=True)
            p = np.where(live[:, None], e_ / np.where(d > 0, d, 1.0), 0.0)
            out[b, h] = p @ v[b, h]
    return out
