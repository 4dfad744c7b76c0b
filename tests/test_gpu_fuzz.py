"""Seeded random cases over the whole request space, every element against the fp64 oracle: mask kind
(dense with / without kv_len, sliding window + global tokens, random block layouts with empty rows),
causal or not, S any multiple of 64 up to 1024, D 64 / 128, fp16 / bf16, and every forward path
(default one launch, unfused, two launches, IR in GEMM2, the paper's standalone IR kernel, SD, GS in
the prologue, key-range split, concurrent), fp32 context or the stored dtype.  The cases are drawn
from a fixed seed, so a failure names a reproducible case."""
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
from tests.test_gpu_parity import TORCH, assert_close  # noqa: E402

PATHS = ["default", "unfused", "two_kernels", "fuse_ir", "ir_kernel", "sd", "gs_prologue", "split_kv", "concurrent"]
N_CASES = 200


def draw(i):
    rng = np.random.Generator(np.random.PCG64(9000 + i))
    kind = ["dense", "window", "block"][int(rng.integers(3))]
    S = 64 * int(rng.integers(1, 17))
    D = [64, 128][int(rng.integers(2))]
    dtype = ["f16", "bf16"][int(rng.integers(2))]
    B, H = int(rng.integers(1, 3)), int(rng.integers(1, 4))
    kw = dict(causal=bool(rng.integers(2)))
    if kind == "dense" and rng.integers(2):
        kw["kv_len"] = [int(x) for x in rng.integers(0, S + 1, size=B)]
    if kind == "window":
        kw["window"] = 2 * int(rng.integers(0, S // 2 + 1))
        kw["n_global"] = int(rng.integers(0, min(S, 80) + 1))
    if kind == "block":
        nb = S // 64
        sets = []
        for _ in range(H):
            rows = []
            for _r in range(nb):
                k = int(rng.integers(0, min(nb, 5) + 1))  # possibly an empty block-row
                rows.append(set(int(c) for c in rng.choice(nb, size=k, replace=False)))
            sets.append(rows)
        kw["layout"] = W.csr_from_sets(64, sets)
    path = PATHS[int(rng.integers(len(PATHS)))]
    out_f32 = bool(rng.integers(2))
    return kind, B, H, S, D, dtype, kw, path, out_f32


@pytest.mark.parametrize("i", range(N_CASES))
def test_fuzz_case(i):
    kind, B, H, S, D, dtype, kw, path, out_f32 = draw(i)
    t, q, k, v = qkv(B, H, S, D, dtype, seed=100 + i)
    scale = 1 / math.sqrt(D)
    mask = {"dense": lambda: sr.dense_mask(kw.get("kv_len")), "block": lambda: sr.block_mask(kw["layout"]),
            "window": lambda: sr.window_mask(kw["window"], kw["n_global"])}[kind]()
    extra = {} if path == "default" else ({"fused": False} if path == "unfused" else {path: True})
    o = sr.call(mask, q, k, v, scale=scale, causal=kw["causal"], out_dtype=torch.float32 if out_f32 else TORCH[dtype],
                **extra)
    torch.cuda.synchronize()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale,
                           oracle_mask(kind, kw.get("kv_len"), kw["causal"], kw.get("layout"), kw.get("window", 0),
                                       kw.get("n_global", 0)))
    what = f"case {i}: {kind} B{B} H{H} S{S} D{D} {dtype} {path} causal={kw['causal']} " \
           f"{ {k_: v_ for k_, v_ in kw.items() if k_ in ('kv_len', 'window', 'n_global')} }"
    assert_close(o.double().cpu().numpy(), ref, dtype, out_f32=out_f32, what=what)


N_BWD = 40


@pytest.mark.parametrize("i", range(N_BWD))
def test_fuzz_backward(i):
    """The training backward (sr_mha_*_bwd) on seeded random requests: O, dQ, dK, dV of every head
    against the fp64 backward oracle (tolerance DESIGN.md R27)."""
    from tests.test_gpu_backward import check, run_bwd
    kind, B, H, S, D, dtype, kw, _path, grads_f32 = draw(10_000 + i)
    got, ref = run_bwd(kind, B, H, S, D, dtype, seed=200 + i, grads_f32=grads_f32, **kw)
    check(got, ref, dtype, grads_f32=grads_f32, what=f"bwd case {i}: {kind} B{B} H{H} S{S} D{D} {dtype} {kw.get('causal')}")


N_F32 = 24


@pytest.mark.parametrize("i", range(N_F32))
def test_fuzz_fp32(i):
    """The fp32 mode (SIMT chain, BASELINE config 1's tolerance 1e-5) on seeded random requests."""
    kind, B, H, S, D, _dtype, kw, _path, _ = draw(20_000 + i)
    t, q, k, v = qkv(B, H, S, D, "f32", seed=300 + i)
    scale = 1 / math.sqrt(D)
    mask = {"dense": lambda: sr.dense_mask(kw.get("kv_len")), "block": lambda: sr.block_mask(kw["layout"]),
            "window": lambda: sr.window_mask(kw["window"], kw["n_global"])}[kind]()
    o = sr.call(mask, q, k, v, scale=scale, causal=kw["causal"])
    torch.cuda.synchronize()
    ref = oracle.attention(t.q64, t.k64, t.v64, scale,
                           oracle_mask(kind, kw.get("kv_len"), kw["causal"], kw.get("layout"), kw.get("window", 0),
                                       kw.get("n_global", 0)))
    assert_close(o.double().cpu().numpy(), ref, "f32", what=f"fp32 case {i}: {kind} B{B} H{H} S{S} D{D}")
