"""Seeded synthetic workloads shared by the oracle tests, the GPU parity tests and bench.py.

This module is the ONLY code both sides of the parity check share (task rule ③). It holds no
arithmetic of the method (no scores, no softmax, no statistics): it draws random numbers,
rounds them to the configuration's storage dtype, and builds the *input* sparsity structures
(the BigBird block layout is an input of the attention layer, not part of the method).

Recipe (DESIGN.md §"Input recipe"):
  * q, k, v ~ i.i.d. N(0, 1) drawn in fp64 from numpy.random.Generator(PCG64(seed)), seeds
    1000+cfg, 2000+cfg, 3000+cfg; rounded to the config dtype with round-to-nearest-even.
    Both sides consume the SAME rounded values (the oracle upcasts them to fp64).
  * scale = 1/sqrt(D) ("divides each element ... by sqrt(D_head)").
  * C2 padding: kv_len = [512, 511, 384, 300, 257, 128, 65, 1] (TriviaQA
    lengths are unavailable, so the list covers full, one-short, tile edges and a single key).
  * C4 BigBird: 64x64 blocks, global blocks {0, nb-1} as full rows and columns, window
    {i-1, i, i+1}, 3 random blocks per block-row drawn without replacement from the
    non-window, non-global blocks with random.Random(h) per head.
  * C5 Longformer: window 512 (|i-j| <= 256) plus 8 symmetric global tokens.
"""
from __future__ import annotations

import math
import random
from dataclasses import dataclass, field
from typing import Optional

import numpy as np

DTYPES = ("f32", "f16", "bf16")


@dataclass
class Config:
    """One BASELINE.json config. ``kind`` selects the entry point: dense / blocksparse / window."""
    idx: int
    name: str
    kind: str
    B: int
    H: int
    S: int
    D: int
    dtype: str
    causal: bool = False
    kv_len: Optional[list] = None
    block: int = 64
    window: int = 0
    n_global: int = 0
    bigbird: Optional[dict] = None

    @property
    def BH(self) -> int:
        return self.B * self.H

    @property
    def scale(self) -> float:
        return 1.0 / math.sqrt(self.D)


# BASELINE.json "configs", in order (1-based index as in SURVEY/BASELINE tables).
CONFIGS = [
    Config(1, "dense_f32_S128", "dense", B=1, H=1, S=128, D=64, dtype="f32"),
    Config(2, "bert_base_pad", "dense", B=8, H=12, S=512, D=64, dtype="f16",
           kv_len=[512, 511, 384, 300, 257, 128, 65, 1]),
    Config(3, "gptneo_causal", "dense", B=4, H=16, S=2048, D=128, dtype="bf16", causal=True),
    Config(4, "bigbird", "blocksparse", B=4, H=12, S=4096, D=64, dtype="f16", block=64,
           bigbird=dict(n_window=3, n_global=2, n_random=3)),
    Config(5, "longformer", "window", B=2, H=12, S=4096, D=64, dtype="f16", window=512, n_global=8),
]


# Second workload of SURVEY NEXT-3 (GPT-Neo's local-attention layers, window 256):
# GPT-Neo's local layers let query i see keys i-255..i, i.e. causal with |i - j| <= 255 -- the
# sliding-window entry with window/2 = 255 (window = 510), no global tokens, at the C3 shape.
GPTNEO_LOCAL = Config(6, "gptneo_local", "window", B=4, H=16, S=2048, D=128, dtype="bf16", causal=True,
                      window=510, n_global=0)
EXTRA_CONFIGS = [GPTNEO_LOCAL]


def config(idx: int) -> Config:
    if idx == GPTNEO_LOCAL.idx:
        return GPTNEO_LOCAL
    return CONFIGS[idx - 1]


# ----------------------------------------------------------------------------- rounding

def _f32_to_bf16_bits(x32: np.ndarray) -> np.ndarray:
    """Round fp32 -> bf16 with round-to-nearest-even; returns uint16 bit patterns."""
    u = x32.astype(np.float32).view(np.uint32).astype(np.uint64)
    nan = np.isnan(x32)
    lsb = (u >> 16) & 1
    r = ((u + 0x7FFF + lsb) >> 16).astype(np.uint16)
    r[nan] = 0x7FC0
    return r


def bf16_bits_to_f64(bits: np.ndarray) -> np.ndarray:
    return (bits.astype(np.uint32) << 16).view(np.float32).astype(np.float64)


def round_to_dtype(x: np.ndarray, dtype: str):
    """Round fp64 values to ``dtype`` (RNE). Returns (storage array, exact fp64 upcast).

    storage: float32 array for f32, float16 array for f16, uint16 bit patterns for bf16.
    """
    if dtype == "f32":
        s = x.astype(np.float32)
        return s, s.astype(np.float64)
    if dtype == "f16":
        s = x.astype(np.float16)
        return s, s.astype(np.float64)
    if dtype == "bf16":
        s = _f32_to_bf16_bits(x.astype(np.float32))
        return s, bf16_bits_to_f64(s)
    raise ValueError(dtype)


# ----------------------------------------------------------------------------- q, k, v

@dataclass
class Tensors:
    """q, k, v in storage form (``*_s``) and as fp64 upcasts (``*_64``), all [B, H, S, D]."""
    q_s: np.ndarray
    k_s: np.ndarray
    v_s: np.ndarray
    q64: np.ndarray
    k64: np.ndarray
    v64: np.ndarray
    dtype: str


def normal(shape, seed: int) -> np.ndarray:
    return np.random.Generator(np.random.PCG64(seed)).standard_normal(shape)


def make_qkv(B, H, S, D, dtype, seed_base: int = 0, heads: Optional[slice] = None) -> Tensors:
    """Seeded N(0,1) q, k, v rounded to ``dtype``. seeds = 1000/2000/3000 + seed_base."""
    shape = (B, H, S, D)
    out = {}
    for name, s0 in (("q", 1000), ("k", 2000), ("v", 3000)):
        x = normal(shape, s0 + seed_base)
        st, x64 = round_to_dtype(x, dtype)
        out[name + "_s"], out[name + "64"] = st, x64
    return Tensors(dtype=dtype, **out)


def make_dout(B, H, S, D, dtype, seed_base: int = 0):
    """Seeded N(0,1) upstream gradient dE/dO (training backward, NEXT-4), rounded to ``dtype``;
    seed 4000 + seed_base.  Returns (storage array, fp64 upcast)."""
    return round_to_dtype(normal((B, H, S, D), 4000 + seed_base), dtype)


def config_tensors(cfg: Config) -> Tensors:
    return make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=cfg.idx)


# ----------------------------------------------------------------------------- layouts (inputs)

@dataclass
class BlockLayout:
    """Block-sparse attention layout: CSR over ``block``-row blocks, one CSR per layout head.

    row_ptr[h, r] are ABSOLUTE offsets into the flat ``col_idx`` (row_ptr[h, 0] is where head h
    starts); column block ids are sorted ascending within a row.
    """
    block: int
    nb: int
    row_ptr: np.ndarray  # int32 [layout_heads, nb + 1]
    col_idx: np.ndarray  # int32 [nnz_total]

    @property
    def layout_heads(self) -> int:
        return self.row_ptr.shape[0]

    def blocks(self, h: int, r: int) -> list:
        return self.col_idx[self.row_ptr[h, r]:self.row_ptr[h, r + 1]].tolist()

    def nnz(self, h: int) -> int:
        return int(self.row_ptr[h, -1] - self.row_ptr[h, 0])


def csr_from_sets(block: int, per_head_rows: list) -> BlockLayout:
    """per_head_rows[h][r] = iterable of column-block ids of block-row r in head h."""
    nb = len(per_head_rows[0])
    rp = np.zeros((len(per_head_rows), nb + 1), dtype=np.int32)
    cols = []
    off = 0
    for h, rows in enumerate(per_head_rows):
        rp[h, 0] = off
        for r, cs in enumerate(rows):
            cs = sorted(set(int(c) for c in cs))
            cols.extend(cs)
            off += len(cs)
            rp[h, r + 1] = off
    return BlockLayout(block=block, nb=nb, row_ptr=rp, col_idx=np.asarray(cols, dtype=np.int32))


def bigbird_layout(H: int, S: int, block: int = 64, n_window: int = 3, n_global: int = 2,
                   n_random: int = 3) -> BlockLayout:
    """BigBird ITC-style layout: global first/last blocks (full rows and
    columns), a 3-block window, 3 random blocks per row from the remaining ones; per-head seed h."""
    assert n_global == 2 and n_window == 3
    nb = S // block
    glob = {0, nb - 1}
    heads = []
    for h in range(H):
        rng = random.Random(h)
        rows = []
        for i in range(nb):
            if i in glob:
                rows.append(range(nb))
                continue
            win = {j for j in (i - 1, i, i + 1) if 0 <= j < nb}
            cand = [j for j in range(nb) if j not in win and j not in glob]
            rnd = rng.sample(cand, min(n_random, len(cand)))
            rows.append(win | glob | set(rnd))
        heads.append(rows)
    return csr_from_sets(block, heads)


def config_layout(cfg: Config) -> Optional[BlockLayout]:
    if cfg.kind != "blocksparse":
        return None
    bb = cfg.bigbird
    return bigbird_layout(cfg.H, cfg.S, cfg.block, bb["n_window"], bb["n_global"], bb["n_random"])


def random_layout(H: int, nb: int, block: int, density: float, seed: int) -> BlockLayout:
    """Random block layout with every block-row non-empty (parity-test input)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    heads = []
    for h in range(H):
        rows = []
        for r in range(nb):
            cs = set(np.nonzero(rng.random(nb) < density)[0].tolist())
            if not cs:
                cs = {int(rng.integers(nb))}
            rows.append(cs)
        heads.append(rows)
    return csr_from_sets(block, heads)


def kv_len_array(cfg: Config) -> Optional[np.ndarray]:
    return None if cfg.kv_len is None else np.asarray(cfg.kv_len, dtype=np.int32)
