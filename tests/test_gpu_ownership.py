"""The §8(b) ownership contract on the GPU (include/sr_mha.h "Ownership"):

  * no device allocation by the library: 100 calls with 100 distinct kv_len vectors (BERT-style
    serving, where the padding mask changes every batch -- PAPER.md L53) leave the device's free
    memory unchanged;
  * no synchronisation: the same calls, enqueued behind a ~1 s device-side spin, all return while
    the spin still runs;
  * graph capture of first-seen masks: 100 calls with masks the library has never seen, captured
    in one CUDA graph, replay to the oracle's results;
  * a replay is self-contained: a graph captured with mask A, replayed after eager calls with mask
    B on the same workspace, still computes mask A (each call re-writes its schedule).
"""
import math
import time

import numpy as np
import pytest

import oracle
from tests.gpu_util import oracle_mask, qkv

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402

B, H, S, D = 4, 2, 384, 64


def _kv_lists(n, seed):
    rng = np.random.Generator(np.random.PCG64(seed))
    seen, out = set(), []
    while len(out) < n:
        kv = tuple(int(x) for x in rng.integers(1, S + 1, size=B))
        if kv not in seen:
            seen.add(kv)
            out.append(list(kv))
    return out


def _ws_max(kvs, **kw):
    return max(sr.workspace_info(sr.dense_mask(kv), B, H, S, D, sr.SR_F16, **kw)["total_bytes"] for kv in kvs)


def test_no_device_allocation_for_new_masks():
    t, q, k, v = qkv(B, H, S, D, "f16", seed=1)
    kvs = _kv_lists(101, seed=1)
    ws = torch.empty(_ws_max(kvs), dtype=torch.uint8, device="cuda")
    out = torch.empty(B, H, S, D, dtype=torch.float16, device="cuda")
    sr.call(sr.dense_mask(kvs[0]), q, k, v, out=out, workspace=ws)  # context, modules, attributes
    torch.cuda.synchronize()
    free0, _ = torch.cuda.mem_get_info()
    for kv in kvs[1:]:
        sr.call(sr.dense_mask(kv), q, k, v, out=out, workspace=ws)
    torch.cuda.synchronize()
    free1, _ = torch.cuda.mem_get_info()
    assert free1 == free0, f"device free memory changed by {free0 - free1} bytes over 100 new masks"


def test_calls_do_not_synchronise():
    t, q, k, v = qkv(B, H, S, D, "f16", seed=2)
    kvs = _kv_lists(100, seed=2)
    ws = torch.empty(_ws_max(kvs), dtype=torch.uint8, device="cuda")
    out = torch.empty(B, H, S, D, dtype=torch.float16, device="cuda")
    sr.call(sr.dense_mask([S] * B), q, k, v, out=out, workspace=ws)
    torch.cuda.synchronize()
    torch.cuda._sleep(2_000_000_000)  # ~1 s of device time at 1.9 GHz
    t0 = time.perf_counter()
    for kv in kvs:
        sr.call(sr.dense_mask(kv), q, k, v, out=out, workspace=ws)
    host_s = time.perf_counter() - t0
    busy = not torch.cuda.current_stream().query()
    torch.cuda.synchronize()
    assert busy, "the stream drained while the calls were enqueued: some call synchronised"
    assert host_s < 0.5, host_s


def test_graph_capture_of_first_seen_masks():
    t, q, k, v = qkv(B, H, S, D, "f16", seed=3)
    kvs = _kv_lists(100, seed=3)
    ws = torch.empty(_ws_max(kvs), dtype=torch.uint8, device="cuda")
    outs = [torch.empty(B, H, S, D, dtype=torch.float32, device="cuda") for _ in kvs]
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for kv, o in zip(kvs, outs):
            sr.call(sr.dense_mask(kv), q, k, v, out=o, out_dtype=torch.float32, workspace=ws)
    for o in outs:
        o.zero_()
    g.replay()
    torch.cuda.synchronize()
    scale = 1 / math.sqrt(D)
    for kv, o in zip(kvs, outs):
        ref = oracle.attention(t.q64, t.k64, t.v64, scale, oracle_mask("dense", kv))
        assert np.abs(o.double().cpu().numpy() - ref).max() <= 1e-2, kv


@pytest.mark.parametrize("train", [False, True])
def test_graph_replay_rewrites_its_schedule(train):
    t, q, k, v = qkv(B, H, S, D, "f16", seed=4)
    kv_a, kv_b = [S, 100, 17, 300], [5, S, 200, 129]
    kw = dict(causal=True, train=True) if train else dict(causal=True)
    ws = torch.empty(_ws_max([kv_a, kv_b], **kw), dtype=torch.uint8, device="cuda")
    o_a = torch.empty(B, H, S, D, dtype=torch.float32, device="cuda")
    o_b = torch.empty_like(o_a)
    sr.call(sr.dense_mask(kv_a), q, k, v, out=o_a, out_dtype=torch.float32, causal=True, workspace=ws)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        sr.call(sr.dense_mask(kv_a), q, k, v, out=o_a, out_dtype=torch.float32, causal=True, workspace=ws)
    o_a.zero_()
    sr.call(sr.dense_mask(kv_b), q, k, v, out=o_b, out_dtype=torch.float32, causal=True, workspace=ws)
    g.replay()
    torch.cuda.synchronize()
    scale = 1 / math.sqrt(D)
    for kv, o in ((kv_a, o_a), (kv_b, o_b)):
        ref = oracle.attention(t.q64, t.k64, t.v64, scale, oracle_mask("dense", kv, causal=True))
        assert np.abs(o.double().cpu().numpy() - ref).max() <= 1e-2, kv


def test_python_binding_checks_buffers():
    """a wrong-sized / wrong-dtype out or gradient is rejected before the C call."""
    t, q, k, v = qkv(1, 1, 128, 64, "f16", seed=5)
    with pytest.raises(ValueError):
        sr.mha_dense(q, k, v, out=torch.empty(1, 1, 128, 64, dtype=torch.float16, device="cuda"),
                     out_dtype=torch.float32)
    with pytest.raises(ValueError):
        sr.mha_dense(q, k, v, out=torch.empty(1, 1, 64, 64, dtype=torch.float16, device="cuda"))
    layer = sr.AttentionTrain(sr.dense_mask(None))
    o = layer.forward(q, k, v)
    with pytest.raises(ValueError):
        layer.backward(torch.ones_like(q), dq=torch.empty(1, 1, 64, 64, dtype=torch.float16, device="cuda"))
    with pytest.raises(ValueError):
        sr.call_bwd(sr.dense_mask(None), q, k[:, :, :64].contiguous(), v, o, torch.ones_like(q), workspace=layer.ws)


PATHS = {"unfused": dict(fused=False), "two_kernels": dict(two_kernels=True), "fuse_ir": dict(fuse_ir=True),
         "ir_kernel": dict(ir_kernel=True), "sd": dict(sd=True), "gs_prologue": dict(gs_prologue=True),
         "split_kv": dict(split_kv=True), "concurrent": dict(concurrent=True)}


@pytest.mark.parametrize("path", list(PATHS))
def test_graph_capture_every_path(path):
    """Every variant path is a self-contained sequence of kernel nodes too: 8 first-seen masks per
    path captured in one graph (workspace sized for the path), replayed, against the oracle."""
    kw = PATHS[path]
    t, q, k, v = qkv(B, H, S, D, "f16", seed=6)
    kvs = _kv_lists(8, seed=list(PATHS).index(path) + 7)
    wmode = dict(fused=kw.get("fused", True), sd=kw.get("sd", False))
    ws = torch.empty(max(sr.workspace_info(sr.dense_mask(kv), B, H, S, D, sr.SR_F16, **wmode)["total_bytes"]
                         for kv in kvs), dtype=torch.uint8, device="cuda")
    outs = [torch.empty(B, H, S, D, dtype=torch.float32, device="cuda") for _ in kvs]
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for kv, o in zip(kvs, outs):
            sr.call(sr.dense_mask(kv), q, k, v, out=o, out_dtype=torch.float32, workspace=ws, causal=True, **kw)
    for o in outs:
        o.zero_()
    g.replay()
    torch.cuda.synchronize()
    scale = 1 / math.sqrt(D)
    for kv, o in zip(kvs, outs):
        ref = oracle.attention(t.q64, t.k64, t.v64, scale, oracle_mask("dense", kv, True))
        assert np.abs(o.double().cpu().numpy() - ref).max() <= 1e-2, (path, kv)
