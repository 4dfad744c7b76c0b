"""fp64 CPU oracle for softmax-recomposed attention -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline / ``--impl reference``
legs may import this package. The product path (``paper_conf_iiswc_choilkha22_b200``) never
imports it and shares no code with it.

``sr_oracle.c`` holds the definitions (see its header for the PAPER.md citations); this module
only compiles it on demand with gcc and marshals numpy arrays through ctypes.

Parity status: every function here is pinned by ``tests/test_oracle_pins.py``
(hand-worked 4x4 examples, closed forms at GPU shapes, invariants, brute force, library routines).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "sr_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

KIND = {"none": 0, "block": 1, "window": 2, "elem": 3}


def build(force: bool = False) -> str:
    """Compile sr_oracle.c -> liboracle.so (plain -O2, no fast-math: exp/max/sum stay IEEE)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-Wall", "-o", tmp, _SRC,
                               "-lm", "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


class _Mask(C.Structure):
    _fields_ = [("kind", C.c_int), ("causal", C.c_int), ("kv_len", C.c_void_p),
                ("block", C.c_int), ("layout_heads", C.c_int), ("row_ptr", C.c_void_p),
                ("col_idx", C.c_void_p), ("window", C.c_int), ("n_global", C.c_int),
                ("elem", C.c_void_p)]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(_LIB)
            dp, ip = C.c_void_p, C.c_int
            L.or_attention.argtypes = [dp, dp, dp, dp, ip, ip, ip, ip, C.c_double, C.POINTER(_Mask), ip]
            L.or_attention.restype = ip
            L.or_attention_rows.argtypes = [dp, dp, dp, ip, ip, ip, ip, C.c_double, C.POINTER(_Mask),
                                            dp, C.c_int64, dp, ip]
            L.or_attention_rows.restype = ip
            L.or_recomposed.argtypes = [dp, dp, dp, dp, ip, ip, ip, ip, C.c_double, C.POINTER(_Mask),
                                        ip, dp, dp, dp, ip]
            L.or_recomposed.restype = ip
            L.or_count_allowed.argtypes = [ip, ip, ip, C.POINTER(_Mask), dp]
            L.or_count_allowed.restype = C.c_int64
            _lib = L
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


class Mask:
    """Mask specification (kept alive while the C call runs).

    kind: "none" | "block" | "window" | "elem"; kv_len: [B] int or None; causal: bool;
    layout: workloads.BlockLayout for "block"; window/n_global for "window";
    elem: uint8 [B*H, S, S] for "elem".
    """

    def __init__(self, kind="none", kv_len=None, causal=False, layout=None, window=0, n_global=0,
                 elem=None):
        self.kv_len = None if kv_len is None else np.ascontiguousarray(kv_len, dtype=np.int32)
        self.row_ptr = self.col_idx = None
        if layout is not None:
            self.row_ptr = np.ascontiguousarray(layout.row_ptr, dtype=np.int32)
            self.col_idx = np.ascontiguousarray(layout.col_idx, dtype=np.int32)
        self.elem = None if elem is None else np.ascontiguousarray(elem, dtype=np.uint8)
        self.c = _Mask(KIND[kind], int(bool(causal)), _ptr(self.kv_len),
                       layout.block if layout is not None else 0,
                       layout.layout_heads if layout is not None else 0,
                       _ptr(self.row_ptr), _ptr(self.col_idx), int(window), int(n_global),
                       _ptr(self.elem))


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def attention(q, k, v, scale, mask: Optional[Mask] = None, nthreads: int = 0, return_threads=False):
    """Textbook attention. q, k, v fp64 [B, H, S, D] -> fp64 [B, H, S, D]."""
    mask = mask or Mask()
    q, k, v = _f64(q), _f64(k), _f64(v)
    B, H, S, D = q.shape
    out = np.empty_like(q)
    nt = lib().or_attention(_ptr(q), _ptr(k), _ptr(v), _ptr(out), B, H, S, D, float(scale),
                            C.byref(mask.c), int(nthreads))
    return (out, nt) if return_threads else out


def attention_rows(q, k, v, scale, rows, mask: Optional[Mask] = None, nthreads: int = 0,
                   return_threads=False):
    """Selected output rows (flat ids bh*S + i) -> fp64 [len(rows), D]."""
    mask = mask or Mask()
    q, k, v = _f64(q), _f64(k), _f64(v)
    B, H, S, D = q.shape
    rows = np.ascontiguousarray(rows, dtype=np.int64)
    out = np.empty((len(rows), D), dtype=np.float64)
    nt = lib().or_attention_rows(_ptr(q), _ptr(k), _ptr(v), B, H, S, D, float(scale),
                                 C.byref(mask.c), _ptr(rows), len(rows), _ptr(out), int(nthreads))
    return (out, nt) if return_threads else out


def recomposed(q, k, v, scale, T, mask: Optional[Mask] = None, nthreads: int = 0):
    """Eq. (2) decomposition (LS, IR, GS, MatMul). Returns (out, m', d', r') with the statistics
    laid out [B*H, ceil(S/T), S]."""
    mask = mask or Mask()
    q, k, v = _f64(q), _f64(k), _f64(v)
    B, H, S, D = q.shape
    nsv = (S + T - 1) // T
    out = np.empty_like(q)
    mp = np.empty((B * H, nsv, S))
    dp = np.empty_like(mp)
    rp = np.empty_like(mp)
    lib().or_recomposed(_ptr(q), _ptr(k), _ptr(v), _ptr(out), B, H, S, D, float(scale),
                        C.byref(mask.c), int(T), _ptr(mp), _ptr(dp), _ptr(rp), int(nthreads))
    return out, mp, dp, rp


def count_allowed(B, H, S, mask: Mask):
    """Number of kept (i, j) elements, total and per head [B*H]."""
    per = np.zeros(B * H, dtype=np.int64)
    tot = lib().or_count_allowed(B, H, S, C.byref(mask.c), _ptr(per))
    return int(tot), per
