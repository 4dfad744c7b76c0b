"""Head sharding of one attention layer across ranks.

The B*H heads of a layer are independent units (the SDA block runs H_num
attention layers in parallel), so a layer shards across GPUs with no exchange step: rank r takes a
contiguous range of the flattened head index g = b*H + h -- one contiguous slice of q, k, v, out in
the [B, H, S, D] layout -- and runs it as a layer of B' = n heads, H' = 1, with the per-head mask
re-packed (kv_len per head, one block layout per head).  Ranges are balanced by tile count
(padding and layouts make per-head work uneven) while staying contiguous.

bench.py --gpus N splits ONE layer this way (strong scaling: layer time = max over ranks) and also
times each shard on one GPU (strong_scaling_shards); tools/multi_gpu_validate.py gathers the output
shards over NCCL for validation (tests/test_dist_gloo.py covers the same logic with gloo on CPU).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Optional

import numpy as np


@dataclass
class Shard:
    g0: int            # first flat head (b*H + h)
    g1: int            # one past the last
    kv_len: Optional[np.ndarray] = None  # per shard head, dense masks with padding
    layout: Optional[object] = None      # block layout with one layout head per shard head

    @property
    def n(self) -> int:
        return self.g1 - self.g0

    @property
    def BH(self):
        """(B', H') of the shard layer: per-head kv_len needs heads on the batch axis (kv_len is
        indexed by b), per-head block layouts need them on the head axis (layouts are indexed by h)."""
        return (1, self.n) if self.layout is not None else (self.n, 1)


@dataclass
class ShardLayout:
    """Block layout re-packed with one layout head per shard head (absolute row_ptr offsets)."""
    block: int
    row_ptr: np.ndarray
    col_idx: np.ndarray

    @property
    def layout_heads(self) -> int:
        return self.row_ptr.shape[0]


def contiguous_ranges(costs, world: int):
    """Split heads 0..len(costs)-1 into `world` contiguous ranges with near-equal total cost
    (greedy prefix cut at multiples of total/world)."""
    c = np.asarray(costs, dtype=np.float64)
    n = len(c)
    cum = np.concatenate([[0.0], np.cumsum(c)])
    cuts = [0]
    for r in range(1, world):
        target = cum[-1] * r / world
        k = int(np.searchsorted(cum, target))
        k = min(max(k, cuts[-1]), n)
        if k > cuts[-1] and abs(cum[k - 1] - target) < abs(cum[k] - target):
            k -= 1
        cuts.append(max(k, cuts[-1]))
    cuts.append(n)
    return [(cuts[r], cuts[r + 1]) for r in range(world)]


def head_costs(B: int, H: int, S: int, T: int = 64, kv_len=None, layout=None, causal: bool = False):
    """Relative work per flat head: its listed (row-block, key-tile) tiles at sub-vector width T (the
    library default T = 64) plus a fixed cost of 1.5 tiles per row-block (Q load, row statistics,
    O store), the same cost model as the library's LPT CTA schedule (abi.cu).  Heads of an unpadded
    dense or windowed layer all cost the same."""
    n_rb = -(-S // 128)  # S % 128 == 64: the last row-block is half inside the head
    fixed = 1.5 * n_rb
    if kv_len is not None:
        def tiles(kv):
            n = 0
            for rb in range(n_rb):
                hi = kv if not causal else min(kv, (rb + 1) * 128)
                n += -(-hi // T) if hi > 0 else 0
            return n
        per_b = [tiles(int(k)) for k in kv_len]
        return [per_b[g // H] + fixed for g in range(B * H)]
    if layout is not None:
        rp = np.asarray(layout.row_ptr)
        ci = np.asarray(layout.col_idx)

        def tiles_lh(lh):  # block-rows 2p, 2p+1 share a 128-row tile over the union of their columns
            n = 0
            for p in range(n_rb):
                cols = set()
                for br in (2 * p, 2 * p + 1):
                    if br >= rp.shape[1] - 1:
                        continue
                    c = ci[rp[lh, br]:rp[lh, br + 1]].tolist()
                    cols.update(x for x in c if not causal or x <= br)
                n += len(cols)
            return n
        per_lh = {}
        out = []
        for g in range(B * H):
            lh = 0 if rp.shape[0] == 1 else g % H
            if lh not in per_lh:
                per_lh[lh] = tiles_lh(lh)
            out.append(per_lh[lh] + fixed)
        return out
    return [1.0] * (B * H)


def make_shard(rank: int, world: int, B: int, H: int, S: int, kv_len=None, layout=None, T: int = 64,
               causal: bool = False, **_mask) -> Shard:
    """Rank `rank`'s shard of the layer (window / n_global / kind in **_mask do not change per-head
    costs: every head of a windowed layer has the same tiles)."""
    g0, g1 = contiguous_ranges(head_costs(B, H, S, T, kv_len, layout, causal), world)[rank]
    sh = Shard(g0, g1)
    if kv_len is not None:
        sh.kv_len = np.asarray([kv_len[g // H] for g in range(g0, g1)], dtype=np.int32)
    if layout is not None:
        nb = S // layout.block
        rp = np.zeros((sh.n, nb + 1), dtype=np.int32)
        cols = []
        for k, g in enumerate(range(g0, g1)):
            lh = 0 if layout.layout_heads == 1 else g % H
            src = np.asarray(layout.row_ptr[lh])
            rp[k, 0] = len(cols)
            for r in range(nb):
                cols.extend(np.asarray(layout.col_idx[src[r]:src[r + 1]]).tolist())
                rp[k, r + 1] = len(cols)
        sh.layout = ShardLayout(layout.block, rp, np.asarray(cols, dtype=np.int32))
    return sh


def shard_view(x, shard: Shard):
    """[B, H, S, D] tensor -> the shard's [B', H', S, D] contiguous slice (a view)."""
    B, H, S, D = x.shape
    return x.reshape(B * H, S, D)[shard.g0:shard.g1].reshape(*shard.BH, S, D)
