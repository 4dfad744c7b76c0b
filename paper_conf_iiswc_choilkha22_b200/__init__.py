"""Python binding of the B200-native softmax-recomposed attention library (libsr_mha.so).

Argument marshalling only: every step of the hot path (GEMM1 + Local Softmax, IR, Global
Scaling + GEMM2, and the unfused baseline) runs in the CUDA kernels behind the C ABI declared in
``include/sr_mha.h``.  PyTorch supplies device memory and the current CUDA stream.  There is no
CPU fallback: if the shared library is missing or a call fails, this module raises.

Entry points (same names as the C ABI, PAPER.md L51-L53 semantics):
    mha_dense(q, k, v, scale=None, kv_len=None, causal=False, ...)
    mha_blocksparse(q, k, v, layout, scale=None, causal=False, ...)
    mha_sliding_window(q, k, v, window, n_global, scale=None, causal=False, ...)
with ``fused=False`` selecting the unfused GEMM -> softmax -> GEMM baseline, and the training
backward (§6, Eq. 3) on the forward's workspace:
    mha_dense_bwd / mha_blocksparse_bwd / mha_sliding_window_bwd (q, k, v, out, dout, ...)
    AttentionTrain(mask): forward() keeps its workspace for backward()
"""
from __future__ import annotations

import ctypes as C
import math
import os
import threading
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SR_MHA_LIB: an experiment build of the same library (build.py --define ... --out PATH)
LIB_PATH = os.environ.get("SR_MHA_LIB") or os.path.join(_HERE, "libsr_mha.so")

SR_OK, SR_ERR_INVALID, SR_ERR_UNSUPPORTED, SR_ERR_WORKSPACE, SR_ERR_CUDA = range(5)
SR_F32, SR_F16, SR_BF16 = 0, 1, 2
SR_E_DENSE, SR_E_BLOCKSPARSE, SR_E_WINDOW = 0, 1, 2

# every symbol include/sr_mha.h declares
EXPORTS = ["sr_mha_dense", "sr_mha_blocksparse", "sr_mha_sliding_window", "sr_mha_dense_unfused",
           "sr_mha_blocksparse_unfused", "sr_mha_sliding_window_unfused", "sr_workspace_bytes",
           "sr_workspace_query", "sr_schedule_stats", "sr_status_string", "sr_last_error",
           "sr_launch_count", "sr_version", "sr_mha_dense_bwd", "sr_mha_blocksparse_bwd",
           "sr_mha_sliding_window_bwd"]
SR_WS_UNFUSED, SR_WS_RECOMPOSED, SR_WS_SD, SR_WS_TRAIN = 0, 1, 2, 3


class SrError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_STATUS = {0: "SR_OK", 1: "SR_ERR_INVALID", 2: "SR_ERR_UNSUPPORTED", 3: "SR_ERR_WORKSPACE", 4: "SR_ERR_CUDA"}


class DenseMask(C.Structure):
    _fields_ = [("kv_len", C.c_void_p)]


class BlockLayoutC(C.Structure):
    _fields_ = [("block", C.c_int32), ("layout_heads", C.c_int32), ("row_ptr", C.c_void_p),
                ("col_idx", C.c_void_p)]


class WindowC(C.Structure):
    _fields_ = [("window", C.c_int32), ("n_global", C.c_int32)]


class Exec(C.Structure):
    _fields_ = [("in_dtype", C.c_int), ("out_dtype", C.c_int), ("workspace", C.c_void_p),
                ("workspace_bytes", C.c_size_t), ("stream", C.c_void_p), ("tile_n", C.c_int32),
                ("flags", C.c_int32)]


class WsInfo(C.Structure):
    _fields_ = [("tile_n", C.c_int32), ("slots_per_head", C.c_int32), ("n_slots", C.c_int64),
                ("xprime_elt_bytes", C.c_int32), ("off_xprime", C.c_size_t), ("off_mprime", C.c_size_t),
                ("off_dprime", C.c_size_t), ("off_rprime", C.c_size_t), ("off_p", C.c_size_t),
                ("off_rowstat", C.c_size_t), ("total_bytes", C.c_size_t), ("off_ds", C.c_size_t),
                ("off_bstat", C.c_size_t), ("off_sched", C.c_size_t), ("sched_bytes", C.c_size_t),
                ("off_partial", C.c_size_t)]


_lib = None
_lock = threading.Lock()


def lib():
    """Load libsr_mha.so (raises if it has not been built -- there is no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise RuntimeError(f"{LIB_PATH} is missing: build it with "
                                   "`python -m paper_conf_iiswc_choilkha22_b200.build`")
            L = C.CDLL(LIB_PATH)
            vp, i, f = C.c_void_p, C.c_int, C.c_float
            sig = [vp, vp, vp, vp, i, i, i, i, f, vp, i, C.POINTER(Exec)]
            for n in EXPORTS[:6]:
                getattr(L, n).argtypes = sig
                getattr(L, n).restype = i
            bsig = [vp, vp, vp, vp, vp, vp, vp, vp, i, i, i, i, f, vp, i, C.POINTER(Exec)]
            for n in ("sr_mha_dense_bwd", "sr_mha_blocksparse_bwd", "sr_mha_sliding_window_bwd"):
                getattr(L, n).argtypes = bsig
                getattr(L, n).restype = i
            L.sr_workspace_bytes.argtypes = [i, i, i, i, i, i, i, vp, i, i]
            L.sr_workspace_bytes.restype = C.c_size_t
            L.sr_workspace_query.argtypes = [i, i, i, i, i, i, i, vp, i, i, C.POINTER(WsInfo)]
            L.sr_workspace_query.restype = i
            L.sr_schedule_stats.argtypes = [i, i, i, i, vp, i, i, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]
            L.sr_schedule_stats.restype = i
            L.sr_status_string.argtypes = [i]
            L.sr_status_string.restype = C.c_char_p
            L.sr_last_error.restype = C.c_char_p
            L.sr_launch_count.restype = C.c_int64
            L.sr_version.restype = C.c_char_p
            _lib = L
    return _lib


def last_error() -> str:
    return lib().sr_last_error().decode()


def launch_count() -> int:
    return int(lib().sr_launch_count())


def _check(st: int):
    if st != SR_OK:
        raise SrError(st, last_error())


# ----------------------------------------------------------------------------- mask descriptors

class _Mask:
    """Holds a C mask descriptor and the host arrays it points to."""

    def __init__(self, entry: int, obj, keep):
        self.entry, self.obj, self.keep = entry, obj, keep

    @property
    def ptr(self):
        return None if self.obj is None else C.cast(C.byref(self.obj), C.c_void_p)


def dense_mask(kv_len=None) -> _Mask:
    if kv_len is None:
        return _Mask(SR_E_DENSE, None, None)
    a = np.ascontiguousarray(np.asarray(kv_len), dtype=np.int32)
    return _Mask(SR_E_DENSE, DenseMask(a.ctypes.data), a)


def block_mask(layout) -> _Mask:
    """layout: object with .block, .row_ptr [layout_heads, nb+1] (absolute offsets), .col_idx."""
    rp = np.ascontiguousarray(layout.row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(layout.col_idx, dtype=np.int32)
    if ci.size == 0:
        ci = np.zeros(1, dtype=np.int32)
    return _Mask(SR_E_BLOCKSPARSE, BlockLayoutC(int(layout.block), int(rp.shape[0]), rp.ctypes.data,
                                                ci.ctypes.data), (rp, ci))


def window_mask(window: int, n_global: int) -> _Mask:
    return _Mask(SR_E_WINDOW, WindowC(int(window), int(n_global)), None)


# ----------------------------------------------------------------------------- queries

def workspace_info(mask: _Mask, B, H, S, D, in_dtype: int, causal=False, tile_n=0, fused=True, sd=False,
                   train=False) -> dict:
    info = WsInfo()
    mode = SR_WS_TRAIN if train else (2 if (sd and fused) else int(fused))
    _check(lib().sr_workspace_query(mask.entry, mode, B, H, S, D, in_dtype,
                                    mask.ptr, int(causal),
                                    int(tile_n), C.byref(info)))
    return {k: getattr(info, k) for k, _ in WsInfo._fields_}


def schedule_stats(mask: _Mask, B, H, S, causal=False, tile_n=0):
    nt, ne = C.c_int64(), C.c_int64()
    _check(lib().sr_schedule_stats(mask.entry, B, H, S, mask.ptr, int(causal), int(tile_n), C.byref(nt),
                                   C.byref(ne)))
    return int(nt.value), int(ne.value)


# ----------------------------------------------------------------------------- torch entry points

def _torch():
    import torch
    return torch


def dtype_code(dt) -> int:
    torch = _torch()
    return {torch.float32: SR_F32, torch.float16: SR_F16, torch.bfloat16: SR_BF16}[dt]


_ws_cache = {}
_ws_lock = threading.Lock()


def _stream_obj(device, stream):
    """The torch stream a call runs on: the current one, or the caller's raw cudaStream_t."""
    torch = _torch()
    if stream is None:
        return torch.cuda.current_stream(device)
    return torch.cuda.ExternalStream(int(stream), device=device)


def _workspace(device, nbytes, st):
    """Default workspace, one per (device, stream): calls on one stream are ordered, so they may share
    it; calls on different streams never do.  Each use is recorded on the call's stream, so a buffer
    dropped when it grows is not handed out again while a kernel on that stream may still use it."""
    torch = _torch()
    key = (device.index if device.index is not None else torch.cuda.current_device(), st.cuda_stream)
    with _ws_lock:
        buf = _ws_cache.get(key)
        if buf is None or buf.numel() < nbytes:
            buf = torch.empty(max(nbytes, 1 << 20), dtype=torch.uint8, device=device)
            _ws_cache[key] = buf
    buf.record_stream(st)
    return buf


def _check_tensor(name, t, shape, dtype, device):
    if not t.is_cuda or t.device != device:
        raise ValueError(f"{name} must be a CUDA tensor on {device}")
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} has shape {tuple(t.shape)}, expected {tuple(shape)}")
    if t.dtype != dtype:
        raise ValueError(f"{name} has dtype {t.dtype}, expected {dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")


def _check_workspace(ws, device, need):
    if not ws.is_cuda or ws.device != device or not ws.is_contiguous():
        raise ValueError(f"workspace must be a contiguous CUDA tensor on {device}")
    if ws.numel() * ws.element_size() < need:
        raise ValueError(f"workspace holds {ws.numel() * ws.element_size()} bytes, the call needs {need}")


_FN = {(SR_E_DENSE, True): "sr_mha_dense", (SR_E_BLOCKSPARSE, True): "sr_mha_blocksparse",
       (SR_E_WINDOW, True): "sr_mha_sliding_window", (SR_E_DENSE, False): "sr_mha_dense_unfused",
       (SR_E_BLOCKSPARSE, False): "sr_mha_blocksparse_unfused",
       (SR_E_WINDOW, False): "sr_mha_sliding_window_unfused"}


SR_RUN_GEMM1, SR_RUN_REDUCE, SR_RUN_GEMM2 = 1, 2, 4
SR_FUSE_IR = 16
SR_DECOMPOSE = 32
SR_IR_KERNEL = 64
SR_ONE_KERNEL = 128
SR_TWO_KERNELS = 256
SR_GS_PROLOGUE = 512
SR_SCHED_RESIDENT = 1024
SR_SPLIT_KV = 2048
SR_CONCURRENT = 4096


def call(mask: _Mask, q, k, v, *, scale=None, causal=False, out_dtype=None, tile_n=0, fused=True,
         out=None, workspace=None, stream=None, stages=0, fuse_ir=False, sd=False, ir_kernel=False,
         one_kernel=False, two_kernels=False, gs_prologue=False, sched_resident=False, split_kv=False,
         concurrent=False):
    """Run one attention layer through the C ABI.  q, k, v: CUDA tensors [B, H, S, D].
    Default (16-bit): GEMM1 + LS with the IR merged inside it, then GS + GEMM2, both in one launch.
    ir_kernel=True selects SR_IR_KERNEL (the paper's layout: a standalone IR kernel writing r');
    fuse_ir=True SR_FUSE_IR (IR folded into GEMM2);
    sd=True SR_DECOMPOSE (decomposition without fusion, the paper's SD, NEXT-1);
    one_kernel=True SR_ONE_KERNEL (GEMM1+LS+IR then GS+GEMM2 per CTA in one launch, T = 64; the
    16-bit default anyway); two_kernels=True SR_TWO_KERNELS (the same chain as two launches);
    gs_prologue=True SR_GS_PROLOGUE (one launch, fp16: Global Scaling in GEMM2's prologue instead of
    accumulator-side); sched_resident=True SR_SCHED_RESIDENT (skip the schedule upload: the workspace
    still holds it from an identical earlier call -- bench.py's per-kernel timing); split_kv=True
    SR_SPLIT_KV (long rows cut into key-range chunks: the paper's three-kernel layout + a combine);
    concurrent=True SR_CONCURRENT (GEMM1 and GEMM2 concurrently in one CTA per SM, D = 128)."""
    torch = _torch()
    if not (q.is_cuda and k.is_cuda and v.is_cuda):
        raise ValueError("q, k, v must be CUDA tensors")
    if q.shape != k.shape or q.shape != v.shape or q.dim() != 4:
        raise ValueError("q, k, v must share the shape [B, H, S, D]")
    if not (q.is_contiguous() and k.is_contiguous() and v.is_contiguous()):
        raise ValueError("q, k, v must be contiguous")
    if q.dtype != k.dtype or q.dtype != v.dtype:
        raise ValueError("q, k, v must share a dtype")
    B, H, S, D = q.shape
    scale = 1.0 / math.sqrt(D) if scale is None else float(scale)
    in_dt = dtype_code(q.dtype)
    out_dtype = q.dtype if out_dtype is None else out_dtype
    if one_kernel and not tile_n:
        tile_n = 64
    if k.device != q.device or v.device != q.device:
        raise ValueError("q, k, v must be on one device")
    if out is None:
        with torch.cuda.device(q.device):
            out = torch.empty((B, H, S, D), dtype=out_dtype, device=q.device)
    else:
        _check_tensor("out", out, (B, H, S, D), out_dtype, q.device)
    wmode = 2 if (sd and fused) else int(fused)
    need = lib().sr_workspace_bytes(mask.entry, wmode, B, H, S, D, in_dt, mask.ptr, int(causal), int(tile_n))
    if need == 0:
        raise SrError(lib().sr_workspace_query(mask.entry, wmode, B, H, S, D, in_dt, mask.ptr, int(causal),
                                               int(tile_n), C.byref(WsInfo())), last_error())
    so = _stream_obj(q.device, stream)
    if workspace is None:
        ws = _workspace(q.device, need, so)
    else:
        ws = workspace
        _check_workspace(ws, q.device, need)
    st = so.cuda_stream
    ex = Exec(in_dt, dtype_code(out_dtype), ws.data_ptr(), ws.numel() * ws.element_size(), st, int(tile_n),
              int(stages) | (SR_FUSE_IR if fuse_ir else 0) | (SR_DECOMPOSE if sd else 0) |
              (SR_IR_KERNEL if ir_kernel else 0) | (SR_ONE_KERNEL if one_kernel else 0) |
              (SR_TWO_KERNELS if two_kernels else 0) | (SR_GS_PROLOGUE if gs_prologue else 0) |
              (SR_SCHED_RESIDENT if sched_resident else 0) | (SR_SPLIT_KV if split_kv else 0) |
              (SR_CONCURRENT if concurrent else 0))
    fn = getattr(lib(), _FN[(mask.entry, bool(fused))])
    with torch.cuda.device(q.device):  # the library launches on the current device
        _check(fn(q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(), B, H, S, D, C.c_float(scale),
                  mask.ptr, int(causal), C.byref(ex)))
    return out


def mha_dense(q, k, v, *, scale=None, kv_len=None, causal=False, **kw):
    return call(dense_mask(kv_len), q, k, v, scale=scale, causal=causal, **kw)


def mha_blocksparse(q, k, v, layout, *, scale=None, causal=False, **kw):
    return call(block_mask(layout), q, k, v, scale=scale, causal=causal, **kw)


def mha_sliding_window(q, k, v, window, n_global, *, scale=None, causal=False, **kw):
    return call(window_mask(window, n_global), q, k, v, scale=scale, causal=causal, **kw)


# ----------------------------------------------------------------------------- training backward

_BWD = {SR_E_DENSE: "sr_mha_dense_bwd", SR_E_BLOCKSPARSE: "sr_mha_blocksparse_bwd",
        SR_E_WINDOW: "sr_mha_sliding_window_bwd"}


def train_workspace(mask: _Mask, q, causal=False, tile_n=0):
    """A workspace sized for forward + backward (SR_WS_TRAIN) for q's shape and dtype."""
    torch = _torch()
    B, H, S, D = q.shape
    info = workspace_info(mask, B, H, S, D, dtype_code(q.dtype), causal=causal, tile_n=tile_n, train=True)
    return torch.empty(info["total_bytes"], dtype=torch.uint8, device=q.device)


def call_bwd(mask: _Mask, q, k, v, out, dout, *, workspace, scale=None, causal=False, tile_n=0, dq=None,
             dk=None, dv=None, stream=None, stages=0, sched_resident=False):
    """Backward of the layer that a preceding ``call(..., workspace=workspace)`` (default mode)
    computed.  out: that forward's output (its dtype is the gradients' dtype); dout: dE/dO in q's
    dtype.  Returns (dq, dk, dv)."""
    torch = _torch()
    if q.dim() != 4 or not q.is_cuda:
        raise ValueError("q must be a CUDA tensor [B, H, S, D]")
    dev = q.device
    for name, t in (("q", q), ("k", k), ("v", v), ("dout", dout)):
        _check_tensor(name, t, q.shape, q.dtype, dev)
    if out.dtype not in (q.dtype, torch.float32):
        raise ValueError("out must have q's dtype or float32 (the forward's out_dtype)")
    _check_tensor("out", out, q.shape, out.dtype, dev)
    B, H, S, D = q.shape
    scale = 1.0 / math.sqrt(D) if scale is None else float(scale)
    with torch.cuda.device(dev):
        dq = torch.empty_like(out) if dq is None else dq
        dk = torch.empty_like(out) if dk is None else dk
        dv = torch.empty_like(out) if dv is None else dv
    for name, t in (("dq", dq), ("dk", dk), ("dv", dv)):
        _check_tensor(name, t, q.shape, out.dtype, dev)
    need = workspace_info(mask, B, H, S, D, dtype_code(q.dtype), causal=causal, tile_n=tile_n,
                          train=True)["total_bytes"]
    _check_workspace(workspace, dev, need)
    st = _stream_obj(dev, stream).cuda_stream
    ex = Exec(dtype_code(q.dtype), dtype_code(out.dtype), workspace.data_ptr(),
              workspace.numel() * workspace.element_size(), st, int(tile_n),
              int(stages) | (SR_SCHED_RESIDENT if sched_resident else 0))
    with torch.cuda.device(dev):
        _check(getattr(lib(), _BWD[mask.entry])(q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(),
                                                dout.data_ptr(), dq.data_ptr(), dk.data_ptr(), dv.data_ptr(), B, H,
                                                S, D, C.c_float(scale), mask.ptr, int(causal), C.byref(ex)))
    return dq, dk, dv


class AttentionTrain:
    """Forward + backward of one attention layer sharing one SR_WS_TRAIN workspace:
        layer = AttentionTrain(dense_mask(kv_len), causal=True)
        o = layer.forward(q, k, v);  dq, dk, dv = layer.backward(dout)"""

    def __init__(self, mask: _Mask, causal=False, scale=None, tile_n=0):
        self.mask, self.causal, self.scale, self.tile_n = mask, causal, scale, tile_n
        self.ws = None

    def forward(self, q, k, v, out_dtype=None, out=None):
        need = workspace_info(self.mask, *q.shape, dtype_code(q.dtype), causal=self.causal, tile_n=self.tile_n,
                              train=True)["total_bytes"]
        if self.ws is None or self.ws.numel() < need or self.ws.device != q.device:
            self.ws = train_workspace(self.mask, q, causal=self.causal, tile_n=self.tile_n)
        self.saved = (q, k, v)
        self.out = call(self.mask, q, k, v, scale=self.scale, causal=self.causal, out_dtype=out_dtype,
                        tile_n=self.tile_n, out=out, workspace=self.ws)
        return self.out

    def backward(self, dout, **kw):
        q, k, v = self.saved
        return call_bwd(self.mask, q, k, v, self.out, dout, workspace=self.ws, scale=self.scale,
                        causal=self.causal, tile_n=self.tile_n, **kw)


def mha_dense_bwd(q, k, v, out, dout, *, workspace, kv_len=None, **kw):
    return call_bwd(dense_mask(kv_len), q, k, v, out, dout, workspace=workspace, **kw)


def mha_blocksparse_bwd(q, k, v, out, dout, layout, *, workspace, **kw):
    return call_bwd(block_mask(layout), q, k, v, out, dout, workspace=workspace, **kw)


def mha_sliding_window_bwd(q, k, v, out, dout, window, n_global, *, workspace, **kw):
    return call_bwd(window_mask(window, n_global), q, k, v, out, dout, workspace=workspace, **kw)
