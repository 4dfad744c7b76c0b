#!/usr/bin/env python
"""bench.py -- attention layers/s and HBM bytes/layer of the softmax-recomposed path vs the in-repo
unfused path on B200 (BASELINE.json "metric").

One step = one attention layer (all B*H heads of the workload config) through the C ABI's default
path: GEMM1 + Local Softmax (+ the IR merge inside GEMM1) -> GS + GEMM2.
The paper's three-kernel layout (standalone IR kernel, SR_IR_KERNEL) and the other variants are
timed in the same run and reported under "variants".  Inputs are seeded synthetic tensors
resident in HBM before the timed region; L2 is flushed (256 MiB write) before every timed step.
Timing: CUDA events on the launching stream, barrier + synchronize around the timed region, max
over ranks.  Multi-GPU (torchrun): every rank runs its own full layer on its own inputs (weak
scaling, no collective on the data path); value = layers of all ranks / max-over-ranks time.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2] [--impl ours|reference]

--impl reference times the fp64 CPU oracle (the only reference this paper-only task has) on a
bounded sample of rows of the same workload, rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
FLUSH_BYTES = 256 << 20
SPIN_CYCLES = 400_000  # ~0.2 ms at 1.97 GHz: device-side head start for the host enqueue (timed())


def describe(cfg):
    m = {"dense": (("padding kv_len=" + str(cfg.kv_len)) if cfg.kv_len else ("causal" if cfg.causal else "none")),
         "blocksparse": "BigBird block 64: 3 window + 2 global + 3 random (622 blocks/head)",
         "window": f"Longformer window {cfg.window} + {cfg.n_global} global"}[cfg.kind]
    return (f"C{cfg.idx} {cfg.name}: B={cfg.B} H={cfg.H} S={cfg.S} D={cfg.D} {cfg.dtype}, mask: {m}")


# ----------------------------------------------------------------------------- clocks

class Clocks:
    """nvidia-smi sampler running DURING the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-i", str(self.idx), "-lms", "200"], stdout=self.f, stderr=subprocess.DEVNULL)
        except OSError:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        self.p.wait()
        self.f.flush()
        rows = [l.split(",") for l in open(self.f.name).read().strip().splitlines() if l.strip()]
        os.unlink(self.f.name)
        if not rows:
            return None
        sm = [float(r[1]) for r in rows if r[1].strip().replace(".", "").isdigit()]
        mx = [float(r[2]) for r in rows if r[2].strip().replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in rows for n, v in zip(names, r[5:9]) if v.strip() == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


# ----------------------------------------------------------------------------- byte model

def alg_bytes(cfg, stored, T, out_bytes=None):
    """Algorithmic HBM bytes per layer of the paper's three-kernel layout
    (SR_IR_KERNEL): Q, K, V, O once; the attention matrix written and read once (recomposed) or
    four times (unfused); m', d' written, read by IR, r' written and read."""
    e = 4 if cfg.dtype == "f32" else 2
    eo = e if out_bytes is None else out_bytes
    bhsd = cfg.BH * cfg.S * cfg.D
    xe = 4 if cfg.dtype == "f32" else 2
    rows_tiles = stored / T  # (row, tile) pairs
    rec = {"gemm1_ls": 2 * bhsd * e + xe * stored + 8 * rows_tiles,
           "ir": 12 * rows_tiles,
           "gs_gemm2": xe * stored + 4 * rows_tiles + bhsd * e + bhsd * eo}
    unf = {"gemm1": 2 * bhsd * e + 2 * stored, "softmax": 4 * stored, "gemm2": 2 * stored + bhsd * e + bhsd * eo}
    return rec, unf


def alg_bytes_ir_in_gemm1(cfg, stored, T):
    """Default path (IR merged in GEMM1): GEMM1 writes X' and m' (no d'), plus (m, 1/d) per query
    row; GEMM2 reads X', m' and the row statistics -- no IR kernel, no r'."""
    e = 4 if cfg.dtype == "f32" else 2
    bhsd = cfg.BH * cfg.S * cfg.D
    rows_tiles = stored / T
    rows = cfg.BH * cfg.S
    return {"gemm1_ls_ir": 2 * bhsd * e + 2 * stored + 4 * rows_tiles + 8 * rows,
            "gs_gemm2": 2 * stored + 4 * rows_tiles + 8 * rows + 2 * bhsd * e}


def alg_bytes_bwd(cfg, stored, T):
    """Training backward (NEXT-4, include/sr_mha.h sr_mha_*_bwd), algorithmic HBM bytes per kernel:
    X' is read twice (dS' kernel, dV kernel), dS' written once and read once (dK; dQ is accumulated
    in the dS' kernel); the dense
    operands once each; per (row, tile) m' read and r' written then read; per row the statistics."""
    e = 2
    bhsd = cfg.BH * cfg.S * cfg.D
    rt = stored / T
    rows = cfg.BH * cfg.S
    return {"prep": 2 * bhsd * e + 28 * rows,
            # dS' kernel with dQ fused: + K read and dQ write, no separate dQ pass over dS'
            "ds": 4 * bhsd * e + 2 * stored + 4 * rt + 12 * rows + 2 * stored + 4 * rt,
            "dk": 2 * stored + 2 * bhsd * e,
            "dv": 2 * stored + 4 * rt + 2 * bhsd * e}


def flops(cfg, stored):
    return 4.0 * cfg.D * stored  # two GEMMs, 2 flops per MAC, over stored score elements


# ----------------------------------------------------------------------------- GPU arm

class Layer:
    def __init__(self, cfg, device, seed_base, sr, torch, tile_n=0):
        self.cfg, self.sr, self.torch = cfg, sr, torch
        self.tile_n = tile_n
        t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=seed_base)
        self.host = {}
        self.dev = {}
        for n in ("q", "k", "v"):
            a = getattr(t, n + "_s")
            if cfg.dtype == "bf16":
                ht = torch.from_numpy(a.view(np.int16).copy()).view(torch.bfloat16)
            else:
                ht = torch.from_numpy(np.ascontiguousarray(a))
            self.host[n] = ht.pin_memory()
            self.dev[n] = self.host[n].to(device)
        tdt = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}[cfg.dtype]
        self.out = torch.empty((cfg.B, cfg.H, cfg.S, cfg.D), dtype=tdt, device=device)
        self.out_host = torch.empty_like(self.out, device="cpu").pin_memory()
        if cfg.kind == "dense":
            self.mask = sr.dense_mask(cfg.kv_len)
        elif cfg.kind == "blocksparse":
            self.mask = sr.block_mask(W.config_layout(cfg))
        else:
            self.mask = sr.window_mask(cfg.window, cfg.n_global)
        self.kw = dict(scale=cfg.scale, causal=cfg.causal)
        in_dt = sr.dtype_code(tdt)
        self.in_dt = in_dt

        def ws_for(**kw):
            info = sr.workspace_info(self.mask, cfg.B, cfg.H, cfg.S, cfg.D, in_dt, causal=cfg.causal, **kw)
            return torch.empty(info["total_bytes"], dtype=torch.uint8, device=device), info["tile_n"]

        # default recomposed path (16-bit: the one-launch kernel, T = 64; fp32: SIMT chain)
        self.ws = {}
        self.ws[True], self.T = ws_for(tile_n=tile_n)
        self.n_tiles, self.stored = sr.schedule_stats(self.mask, cfg.B, cfg.H, cfg.S, causal=cfg.causal, tile_n=self.T)
        if cfg.dtype != "f32":
            # two-launch variants (SR_TWO_KERNELS, SR_FUSE_IR, SR_IR_KERNEL) at their tuned T (128; 64 for
            # block-sparse), the unfused baseline and SD at the library default for them
            self.T2 = 64 if cfg.kind == "blocksparse" else 128
            self.ws["t2"], _ = ws_for(tile_n=self.T2)
            _, self.stored2 = sr.schedule_stats(self.mask, cfg.B, cfg.H, cfg.S, causal=cfg.causal, tile_n=self.T2)
            self.ws[False], self.Tu = ws_for(fused=False)
            _, self.stored_u = sr.schedule_stats(self.mask, cfg.B, cfg.H, cfg.S, causal=cfg.causal, tile_n=self.Tu)
            self.ws["sd"], self.Tsd = ws_for(sd=True)

    def setup_train(self, seed_base):
        """Training (NEXT-4): dE/dO, gradient buffers and an SR_WS_TRAIN workspace."""
        cfg, torch, sr = self.cfg, self.torch, self.sr
        do_s, _ = W.make_dout(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=seed_base)
        if cfg.dtype == "bf16":
            self.dout = torch.from_numpy(do_s.view(np.int16).copy()).view(torch.bfloat16).to(self.out.device)
        else:
            self.dout = torch.from_numpy(np.ascontiguousarray(do_s)).to(self.out.device)
        info = sr.workspace_info(self.mask, cfg.B, cfg.H, cfg.S, cfg.D, sr.dtype_code(self.dout.dtype),
                                 causal=cfg.causal, tile_n=self.tile_n, train=True)
        self.ws_train = torch.empty(info["total_bytes"], dtype=torch.uint8, device=self.out.device)
        self.grads = [torch.empty_like(self.out) for _ in range(3)]

    def fwd_train(self):
        d = self.dev
        return self.sr.call(self.mask, d["q"], d["k"], d["v"], out=self.out, workspace=self.ws_train,
                            tile_n=self.tile_n, **self.kw)

    def bwd(self, stages=0):
        d = self.dev
        dq, dk, dv = self.grads
        return self.sr.call_bwd(self.mask, d["q"], d["k"], d["v"], self.out, self.dout, workspace=self.ws_train,
                                dq=dq, dk=dk, dv=dv, stages=stages, tile_n=self.tile_n, **self.kw)

    def train_step(self):
        self.fwd_train()
        self.bwd()

    def run(self, fused=True, stages=0, q=None, k=None, v=None, fuse_ir=False, sd=False, ir_kernel=False,
            two_kernels=False, gs_prologue=False):
        d = self.dev
        two = fuse_ir or ir_kernel or two_kernels
        if sd:
            ws, tn = self.ws["sd"], 0
        elif not fused:
            ws, tn = self.ws[False], 0
        elif two:
            ws, tn = self.ws["t2"], self.T2
        else:
            ws, tn = self.ws[True], self.tile_n
        return self.sr.call(self.mask, q if q is not None else d["q"], k if k is not None else d["k"],
                            v if v is not None else d["v"], out=self.out, fused=fused, stages=stages,
                            workspace=ws, tile_n=tn, fuse_ir=fuse_ir, sd=sd, ir_kernel=ir_kernel,
                            two_kernels=two_kernels, gs_prologue=gs_prologue, **self.kw)


def e2e_pipelined(torch, L, steps, warmup, nbuf=2):
    """End-to-end throughput through the public API: K steps, each copying its q/k/v from pinned host
    memory, running the layer and reading its output back to pinned host memory. Three streams
    (copy-in, compute, copy-out) with double-buffered device inputs/outputs, so step i+1's H2D and
    step i-1's D2H overlap step i's layer (PCIe is full duplex). Every step still moves all its bytes.
    Returns device ms per step (events around the whole K-step region on the compute stream)."""
    comp = torch.cuda.current_stream()
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    bufs = [{n: torch.empty_like(L.dev[n]) for n in ("q", "k", "v")} for _ in range(nbuf)]
    outs = [torch.empty_like(L.out) for _ in range(nbuf)]
    hosts = [torch.empty_like(L.out_host).pin_memory() for _ in range(nbuf)]
    ws = L.ws[True]

    def region(n):
        comp_done = [None] * n
        out_done = [None] * n
        start = torch.cuda.Event(enable_timing=True)
        end = torch.cuda.Event(enable_timing=True)
        comp.record_event(start)
        s_in.wait_event(start)
        for i in range(n):
            b = i % nbuf
            with torch.cuda.stream(s_in):
                if i >= nbuf:
                    s_in.wait_event(comp_done[i - nbuf])  # layer i-nbuf finished reading this input set
                for nm in ("q", "k", "v"):
                    bufs[b][nm].copy_(L.host[nm], non_blocking=True)
                ready = torch.cuda.Event()
                s_in.record_event(ready)
            comp.wait_event(ready)
            if i >= nbuf:
                comp.wait_event(out_done[i - nbuf])  # D2H of step i-nbuf finished reading this output
            L.sr.call(L.mask, bufs[b]["q"], bufs[b]["k"], bufs[b]["v"], out=outs[b], workspace=ws,
                      tile_n=L.tile_n, **L.kw)
            comp_done[i] = torch.cuda.Event()
            comp.record_event(comp_done[i])
            s_out.wait_event(comp_done[i])
            with torch.cuda.stream(s_out):
                hosts[b].copy_(outs[b], non_blocking=True)
                out_done[i] = torch.cuda.Event()
                s_out.record_event(out_done[i])
        comp.wait_event(out_done[n - 1])
        comp.record_event(end)
        return start, end

    region(max(warmup, nbuf))
    torch.cuda.synchronize()
    torch.cuda._sleep(SPIN_CYCLES)
    a, b = region(steps)
    torch.cuda.synchronize()
    # every step computed the same layer from the same host inputs: the pipelined result read back
    # to the host must equal the device path's output bit for bit (the kernels are deterministic)
    L.run()
    torch.cuda.synchronize()
    same = all(torch.equal(h, L.out.cpu()) for h in hosts)
    return a.elapsed_time(b) / steps, same


def timed(torch, fn, steps, warmup, flush, per_step_pre=None):
    """W warm-up + K timed steps; L2 flushed before each; returns per-step device ms list."""
    ev = []
    for s in range(warmup + steps):
        if flush is not None:
            flush[0].zero_()  # write 256 MiB (evicts everything) ...
            flush[1].sum()  # ... then read another 256 MiB so L2 starts the step clean, not dirty
        if per_step_pre:
            per_step_pre()
        # keep the GPU busy (outside the timed region) while the host enqueues the step, so host-side
        # launch latency (ctypes marshalling, the clock-sampling thread) never shows up as idle device
        # time between the two events
        torch.cuda._sleep(SPIN_CYCLES)
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        if s >= warmup:
            ev.append((a, b))
    torch.cuda.synchronize()
    return [a.elapsed_time(b) for a, b in ev]


L2_BYTES = 126 << 20


def rotation_sets(cfg, device, rank, sr, torch, L, tile_n):
    """Independent (q, k, v, out, workspace) sets for back-to-back timing: enough of them that the
    data cycled through between two uses of a set exceeds 2x the L2, so no step finds its inputs or
    its X' in L2 (the 'inputs larger than L2' form of the no-warm-cache rule)."""
    per = sum(t.numel() * t.element_size() for t in (L.dev["q"], L.dev["k"], L.dev["v"], L.out)) + L.ws[True].numel()
    n = max(2, min(8, math.ceil(2 * L2_BYTES / per)))
    sets = [L] + [Layer(cfg, device, seed_base=cfg.idx + 1000 * rank + 100 * i, sr=sr, torch=torch, tile_n=tile_n)
                  for i in range(1, n)]
    return sets, n * per


def steps_graph(torch, fns, K):
    """One CUDA graph of K back-to-back layer calls cycling through fns (each a call on its own set)."""
    for f in fns:
        f()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for i in range(K):
            fns[i % len(fns)]()
    torch.cuda.synchronize()
    return g


def timed_steps(torch, g, K, warmup, reps=3):
    """Device ms per layer of K back-to-back layers (events around the whole graph replay)."""
    for _ in range(max(1, warmup // K + 1)):
        g.replay()
    torch.cuda.synchronize()
    ev = []
    for _ in range(reps):
        torch.cuda._sleep(SPIN_CYCLES)
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        ev.append((a, b))
    torch.cuda.synchronize()
    return [a.elapsed_time(b) / K for a, b in ev]


def capture(torch, fn):
    """CUDA graph of one call of fn.  The library's launches are capturable once a call with the
    same mask has built its schedule (include/sr_mha.h); replaying the graph runs exactly the same
    kernels with the same arguments, without the per-launch host and scheduling overhead (the
    deployment form of a layer; `eager` numbers are reported beside it)."""
    fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fn()
    torch.cuda.synchronize()
    return g


def dist_max(torch, x, world):
    if world == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    return float(t.item())


def barrier(torch, world):
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()


def load_ncu_traffic():
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        try:
            return json.load(open(p))
        except ValueError:
            return {}
    return {}


def gpu_arm(args, rank, world, local_rank):
    import torch
    import paper_conf_iiswc_choilkha22_b200 as sr
    torch.cuda.set_device(local_rank)
    device = torch.device("cuda", local_rank)
    sr.lib()
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {}
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    peak_src = "MEASURED_PEAKS.json hbm_gbs (measured)" if "hbm_gbs" in peaks else "fallback 6650 GB/s (B200_PROFILING.md)"
    cfg = W.config(args.config)
    flush = None if args.no_flush else (torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=device),
                                        torch.ones(FLUSH_BYTES // 4, dtype=torch.float32, device=device))
    L = Layer(cfg, device, seed_base=cfg.idx + 1000 * rank, sr=sr, torch=torch, tile_n=args.tile_n)
    K, Wm = args.steps, args.warmup

    # ---- headline: K back-to-back recomposed layers (C ABI calls captured in one CUDA graph),
    # cycling through input / workspace sets whose footprint exceeds 2x L2; inputs resident in HBM
    L.run()
    n0 = sr.launch_count()
    L.run()
    launches_per_layer = sr.launch_count() - n0
    sets, rot_bytes = rotation_sets(cfg, device, rank, sr, torch, L, args.tile_n)
    g_tp = steps_graph(torch, [x.run for x in sets], K)
    barrier(torch, world)
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    phys = vis.split(",")[local_rank] if vis else str(local_rank)
    clk = Clocks(phys)
    clk.start()
    t_end = time.perf_counter() + 0.8  # keep the GPU under this load while nvidia-smi samples
    while time.perf_counter() < t_end:
        timed_steps(torch, g_tp, K, 0, reps=2)
    ms_rec = timed_steps(torch, g_tp, K, Wm, reps=5)
    launches = launches_per_layer * K
    clocks = clk.stop()
    barrier(torch, world)
    ms_step = dist_max(torch, statistics.mean(ms_rec), world)
    step_stats = {"min": round(min(ms_rec), 5), "median": round(statistics.median(ms_rec), 5),
                  "max": round(max(ms_rec), 5)}
    # one layer alone: an L2 flush before each step, events around the single call
    ms_cold = dist_max(torch, statistics.mean(timed(torch, L.run, K, Wm, flush)), world)

    # ---- unfused in-repo baseline (same tiles, same skipping)
    ms_unf = None
    kern_unf = {}
    f32 = cfg.dtype == "f32"
    if f32:
        hb = alg_bytes(cfg, L.stored, L.T)[0]
    else:
        hb = alg_bytes_ir_in_gemm1(cfg, L.stored, L.T)  # the one-launch kernel moves both kernels' bytes
        unf_b = alg_bytes(cfg, L.stored_u, L.Tu)[1]
        barrier(torch, world)
        g_unf = steps_graph(torch, [(lambda x=x: x.run(fused=False)) for x in sets], K)
        ms_unf = dist_max(torch, statistics.mean(timed_steps(torch, g_unf, K, Wm)), world)
        ms_unf_cold = dist_max(torch, statistics.mean(timed(torch, lambda: L.run(fused=False), K, Wm, flush)), world)
        for name, bit in (("gemm1", 1), ("softmax", 2), ("gemm2", 4)):
            t = statistics.mean(timed(torch, lambda b=bit: L.run(fused=False, stages=b), K, Wm, flush))
            kern_unf[name] = {"us": round(t * 1e3, 3), "alg_bytes": int(unf_b[name]),
                              "GB/s": round(unf_b[name] / (t * 1e-3) / 1e9, 1)}

    # ---- variants (two launches and more): the same chain as two kernels (SR_TWO_KERNELS), the IR
    # folded into GEMM2 (SR_FUSE_IR, NEXT-2), the paper's three-kernel layout (SR_IR_KERNEL), SD (NEXT-1)
    variants = None
    if not f32:
        def graph_ms(**kw):
            g = capture(torch, lambda: L.run(**kw))
            return dist_max(torch, statistics.mean(timed(torch, g.replay, K, Wm, flush)), world)

        def stage_us(bit, **kw):
            L.run(**kw)
            return statistics.mean(timed(torch, lambda: L.run(stages=bit, **kw), K, Wm, flush)) * 1e3

        b2 = alg_bytes_ir_in_gemm1(cfg, L.stored2, L.T2)
        r2 = alg_bytes(cfg, L.stored2, L.T2)[0]
        rt2 = L.stored2 / L.T2
        g_two = steps_graph(torch, [(lambda x=x: x.run(two_kernels=True)) for x in sets], K)
        ms_two_tp = dist_max(torch, statistics.mean(timed_steps(torch, g_two, K, Wm)), world)
        ms_two, ms_fir, ms_irk, ms_sd = (graph_ms(two_kernels=True), graph_ms(fuse_ir=True),
                                         graph_ms(ir_kernel=True), graph_ms(sd=True))
        kern_two = {n: stage_us(bit, two_kernels=True) for n, bit in (("gemm1_ls_ir", 1), ("gs_gemm2", 4))}
        kern_irk = {n: stage_us(bit, ir_kernel=True) for n, bit in (("gemm1_ls", 1), ("ir", 2), ("gs_gemm2_rprime", 4))}
        irk_b = {"gemm1_ls": r2["gemm1_ls"], "ir": r2["ir"], "gs_gemm2_rprime": r2["gs_gemm2"]}

        def kd(times, nbytes):
            return {n: {"us": round(t, 3), "alg_bytes": int(nbytes[n]), "GB/s": round(nbytes[n] / (t * 1e-6) / 1e9, 1)}
                    for n, t in times.items()}

        variants = {
            "two_kernels": {"what": f"the same chain as two launches: GEMM1+LS+IR -> GS+GEMM2 (SR_TWO_KERNELS, T={L.T2})",
                            "value": round(world * 1e3 / ms_two, 2), "ms_per_step": round(ms_two, 5),
                            "back_to_back": {"value": round(world * 1e3 / ms_two_tp, 2), "ms_per_step": round(ms_two_tp, 5)},
                            "alg_bytes": int(sum(b2.values())), "kernels": kd(kern_two, b2)},
            "fused_ir": {"what": f"IR folded into GS+GEMM2 (SURVEY NEXT-2, 2 kernels, T={L.T2})",
                         "value": round(world * 1e3 / ms_fir, 2), "ms_per_step": round(ms_fir, 5),
                         "alg_bytes": int(sum(r2.values()) - 4 * rt2)},
            "ir_kernel": {"what": "the paper's three-kernel layout: GEMM1+LS -> standalone IR kernel (writes r') -> "
                                  f"GS+GEMM2 (SR_IR_KERNEL, PAPER.md L165-L173, T={L.T2})",
                          "value": round(world * 1e3 / ms_irk, 2), "ms_per_step": round(ms_irk, 5),
                          "alg_bytes": int(sum(r2.values())), "kernels": kd(kern_irk, irk_b)},
            "sd": {"what": f"decomposition without fusion: GEMM1 -> LS -> IR -> GS -> GEMM2 (PAPER.md SD, NEXT-1, T={L.Tsd})",
                   "value": round(world * 1e3 / ms_sd, 2), "ms_per_step": round(ms_sd, 5),
                   "alg_bytes": int(sum(unf_b.values()) + 4 * L.stored_u + 24 * L.stored_u / L.Tu)}}
        L.run()

    # ---- the dominant kernel of the default path: the one-launch kernel IS the layer (16-bit); the
    # fp32 SIMT chain is timed per kernel with stage-selected launches
    kern = {}
    if f32:
        for name, bit in (("gemm1_ls", 1), ("ir", 2), ("gs_gemm2", 4)):
            t = statistics.mean(timed(torch, lambda b=bit: L.run(stages=b), K, Wm, flush))
            kern[name] = {"us": round(t * 1e3, 3), "alg_bytes": int(hb[name]), "GB/s": round(hb[name] / (t * 1e-3) / 1e9, 1)}
    else:  # one launch per layer: its average launch duration over the back-to-back timed region
        nb = sum(hb.values())
        kern["sr_layer_one_kernel"] = {"us": round(ms_step * 1e3, 3), "alg_bytes": int(nb),
                                       "GB/s": round(nb / (ms_step * 1e-3) / 1e9, 1),
                                       "us_single_layer_cold": round(ms_cold * 1e3, 3)}

    # ---- training: forward + backward of the layer on one SR_WS_TRAIN workspace
    train = None
    if cfg.dtype != "f32":
        L.setup_train(cfg.idx + 1000 * rank)
        L.train_step()
        g_tr = capture(torch, L.train_step)
        ms_tr = dist_max(torch, statistics.mean(timed(torch, g_tr.replay, K, Wm, flush)), world)
        g_bw = capture(torch, L.bwd)
        ms_bw = dist_max(torch, statistics.mean(timed(torch, g_bw.replay, K, Wm, flush)), world)
        ms_tr_eager = statistics.mean(timed(torch, L.train_step, K, Wm, flush))
        bb = alg_bytes_bwd(cfg, L.stored, L.T)
        kern_bw = {}
        for name, bit, keys in (("prep_ds_dq", 1, ("prep", "ds")), ("dk_dv", 4, ("dk", "dv"))):
            t = statistics.mean(timed(torch, lambda b=bit: L.bwd(stages=b), K, Wm, flush))
            nb = sum(bb[k_] for k_ in keys)
            kern_bw[name] = {"us": round(t * 1e3, 3), "alg_bytes": int(nb), "GB/s": round(nb / (t * 1e-3) / 1e9, 1)}
        train = {"what": "training step = forward (default path) + backward (sr_mha_*_bwd: row statistics, "
                         "dS' = scale*y*(dO V^T - delta) with y = X' r' recomposed per tile (Eq. 3), dQ = dS' K, "
                         "dK = dS'^T Q, dV = y^T dO); L2 flushed before every step",
                 "fwd_bwd_per_s": round(world * 1e3 / ms_tr, 2), "fwd_bwd_ms": round(ms_tr, 5),
                 "fwd_bwd_ms_eager": round(ms_tr_eager, 5),
                 "bwd_ms": round(ms_bw, 5), "alg_bytes_bwd": int(sum(bb.values())),
                 "bwd_hbm_GBps": round(sum(bb.values()) / (ms_bw * 1e-3) / 1e9, 1), "kernels": kern_bw}

    # ---- end to end through the public API: pinned host -> device, layer, device -> host
    h2d = sum(L.host[n].numel() * L.host[n].element_size() for n in ("q", "k", "v"))
    d2h = L.out.numel() * L.out.element_size()
    qd, kd, vd = (torch.empty_like(L.dev[n]) for n in ("q", "k", "v"))

    def e2e_step():
        qd.copy_(L.host["q"], non_blocking=True)
        kd.copy_(L.host["k"], non_blocking=True)
        vd.copy_(L.host["v"], non_blocking=True)
        L.run(q=qd, k=kd, v=vd)
        L.out_host.copy_(L.out, non_blocking=True)

    barrier(torch, world)
    ms_e2e_serial = dist_max(torch, statistics.mean(timed(torch, e2e_step, K, Wm, flush)), world)
    ms_e2e, e2e_same = e2e_pipelined(torch, L, K, Wm)
    ms_e2e = dist_max(torch, ms_e2e, world)

    # ---- other configs (same run, fewer steps): layers/s and bytes, recomposed vs unfused
    others = {}
    if args.all_configs and world == 1:
        for c2 in W.CONFIGS:
            if c2.idx == cfg.idx:
                continue
            L2 = Layer(c2, device, seed_base=c2.idx, sr=sr, torch=torch)
            sets2, _ = rotation_sets(c2, device, 0, sr, torch, L2, 0)
            g2 = steps_graph(torch, [x.run for x in sets2], 10)
            tr = statistics.mean(timed_steps(torch, g2, 10, 3))
            r2 = alg_bytes(c2, L2.stored, L2.T)[0]
            if c2.dtype != "f32":
                r2 = alg_bytes_ir_in_gemm1(c2, L2.stored, L2.T)
                u2 = alg_bytes(c2, L2.stored_u, L2.Tu)[1]
            ent = {"layers_per_s": round(1e3 / tr, 1), "ms": round(tr, 4),
                   "alg_bytes_recomposed": int(sum(r2.values()))}
            if c2.dtype != "f32":
                g2 = steps_graph(torch, [(lambda x=x: x.run(fused=False)) for x in sets2], 10)
                tu = statistics.mean(timed_steps(torch, g2, 10, 3))
                ent.update({"unfused_layers_per_s": round(1e3 / tu, 1), "alg_bytes_unfused": int(sum(u2.values())),
                            "byte_reduction": round(1 - sum(r2.values()) / sum(u2.values()), 4),
                            "speedup_vs_unfused": round(tu / tr, 3)})
            ent["hbm_GBps_recomposed"] = round(sum(r2.values()) / (tr * 1e-3) / 1e9, 1)
            if c2.dtype != "f32":
                g2 = steps_graph(torch, [(lambda x=x: x.run(two_kernels=True)) for x in sets2], 10)
                tw = statistics.mean(timed_steps(torch, g2, 10, 3))
                ent["two_kernels_layers_per_s"] = round(1e3 / tw, 1)
                g2 = capture(torch, lambda: L2.run(fuse_ir=True))
                tf = statistics.mean(timed(torch, g2.replay, 10, 3, flush))
                ent["fused_ir_layers_per_s"] = round(1e3 / tf, 1)
                g2 = capture(torch, lambda: L2.run(ir_kernel=True))
                tg = statistics.mean(timed(torch, g2.replay, 10, 3, flush))
                ent["ir_kernel_layers_per_s"] = round(1e3 / tg, 1)
            if c2.dtype != "f32":
                L2.setup_train(c2.idx)
                g2 = capture(torch, L2.train_step)
                tt = statistics.mean(timed(torch, g2.replay, 10, 3, flush))
                g2 = capture(torch, L2.bwd)
                tb = statistics.mean(timed(torch, g2.replay, 10, 3, flush))
                bb2 = alg_bytes_bwd(c2, L2.stored, L2.T)
                ent.update({"train_fwd_bwd_ms": round(tt, 4), "bwd_ms": round(tb, 4),
                            "bwd_hbm_GBps": round(sum(bb2.values()) / (tb * 1e-3) / 1e9, 1)})
            others[f"C{c2.idx}"] = ent
            del L2, sets2, g2
            torch.cuda.empty_cache()

    if rank != 0:
        return None
    dom = max(kern, key=lambda n: kern[n]["us"])
    ncu = load_ncu_traffic().get(f"C{cfg.idx}", {})
    achieved = kern[dom]["alg_bytes"] / (kern[dom]["us"] * 1e-6) / 1e9
    value = world * 1e3 / ms_step
    res = {
        "metric": METRIC,
        "value": round(value, 2),
        "unit": "layers/s",
        "n_gpus": world, "steps": K, "warmup": Wm,
        "ms_per_step": round(ms_step, 5),
        "timing": f"K back-to-back layer calls (C ABI, captured in one CUDA graph) between two events, over "
                  f"{len(sets)} rotating input/workspace sets ({rot_bytes / 2**20:.0f} MiB > 2x L2, so no step finds its "
                  "data in L2); ms_per_step = region time / K, mean of 5 regions (step_ms: min/median/max); "
                  "single_layer_cold = one call between events with a 256 MiB L2 flush before it; variants and "
                  "training are single-call CUDA-graph replays with the flush",
        "step_ms": step_stats,
        "single_layer_cold": {"value": round(world * 1e3 / ms_cold, 2), "ms_per_step": round(ms_cold, 5)},
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": cfg.dtype,
        "data": "synthetic (seeded N(0,1) q/k/v rounded to dtype; no datasets or weights needed)",
        "config": {"workload": describe(cfg), "B": cfg.B, "H": cfg.H, "S": cfg.S, "D": cfg.D, "T": L.T,
                   "tiles": L.n_tiles, "stored_score_elems": L.stored,
                   "l2": f"inputs larger than L2: {len(sets)} rotating sets, {rot_bytes / 2**20:.0f} MiB cycled between uses of a set; "
                         "single-layer and variant timings flush L2 (256 MiB write + 256 MiB read) before each step",
                   "parallelism": f"dp{world} (weak: each rank runs its own full layer on its own inputs)"},
        "hbm_bytes_per_layer": None if f32 else {
            "recomposed_alg": int(sum(hb.values())), "unfused_alg": int(sum(unf_b.values())),
            "reduction_alg": round(1 - sum(hb.values()) / sum(unf_b.values()), 4),
            "recomposed_ncu": ncu.get("recomposed_dram_bytes"), "unfused_ncu": ncu.get("unfused_dram_bytes")},
        "unfused": None if ms_unf is None else {"value": round(world * 1e3 / ms_unf, 2), "ms_per_step": round(ms_unf, 5),
                                                "speedup_recomposed_vs_unfused": round(ms_unf / ms_step, 3),
                                                "single_layer_cold_ms": round(ms_unf_cold, 5),
                                                "T": L.Tu, "kernels": kern_unf},
        "variants": variants,
        "kernels": kern,
        "roofline": {"kernel": dom, "bound": "hbm", "achieved": round(achieved, 1), "peak": hbm_peak, "unit": "GB/s",
                     "frac": round(achieved / hbm_peak, 4), "traffic": ncu.get(f"{dom}_dram_bytes"),
                     "peak_source": peak_src,
                     "tensor_frac": round(flops(cfg, L.stored) / (ms_step * 1e-3) / 1e12 / peaks.get("bf16_tflops", 1590.0), 4)},
        "e2e": {"value": round(world * 1e3 / ms_e2e, 2), "unit": "layers/s", "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": int(d2h), "ms_per_step": round(ms_e2e, 5),
                "how": "K steps through the public API, each H2D of its q/k/v from pinned host memory, the "
                       "layer, D2H of its output; copy-in / compute / copy-out streams, double-buffered",
                "output_bitwise_equal_device_path": bool(e2e_same),
                "pcie_GBps": round((h2d + d2h) / (ms_e2e * 1e-3) / 1e9, 1),
                "single_step_serial": {"value": round(world * 1e3 / ms_e2e_serial, 2),
                                       "ms_per_step": round(ms_e2e_serial, 5)}},
        "gpu_launches": int(launches),
        "training": train,
        "clocks": clocks,
    }
    if others:
        res["all_configs"] = others
    return res


# ----------------------------------------------------------------------------- CPU (oracle) arm

def oracle_sample(cfg, target_s, seed=0):
    """Time the fp64 oracle on a bounded random sample of rows; returns (layers/s, rows, secs, threads)."""
    import oracle
    t = W.config_tensors(cfg)
    m = oracle_mask_for(cfg)
    rng = np.random.Generator(np.random.PCG64(seed))
    total = cfg.BH * cfg.S
    probe = rng.integers(0, total, size=min(64, total))
    t0 = time.perf_counter()
    _, nt = oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, probe, m, return_threads=True)
    dt = max(time.perf_counter() - t0, 1e-4)
    n = int(min(total, max(64, len(probe) * target_s / dt)))
    return t, m, n, nt


def oracle_mask_for(cfg):
    import oracle
    if cfg.kind == "dense":
        return oracle.Mask(kv_len=cfg.kv_len, causal=cfg.causal)
    if cfg.kind == "blocksparse":
        return oracle.Mask(kind="block", layout=W.config_layout(cfg), causal=cfg.causal)
    return oracle.Mask(kind="window", window=cfg.window, n_global=cfg.n_global, causal=cfg.causal)


def cpu_baseline(cfg, target_s=10.0):
    import oracle
    t, m, n, nt = oracle_sample(cfg, target_s)
    rng = np.random.Generator(np.random.PCG64(1))
    done, reps = 0, 0
    t0 = time.perf_counter()
    while True:  # repeat the bounded sample until ~target_s of CPU work has been timed
        rows = rng.integers(0, cfg.BH * cfg.S, size=n)
        oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, m)
        done += n
        reps += 1
        dt = time.perf_counter() - t0
        if dt >= 0.9 * target_s:
            break
    frac = done / (cfg.BH * cfg.S)
    return {"value": round(frac / dt, 6), "unit": "layers/s", "cores": nt, "kind": "oracle",
            "sample": f"{reps} x {n} uniformly drawn query rows of {cfg.BH * cfg.S} ({frac:.4f} layers in total), "
                      f"{dt:.2f} s, fp64 textbook attention, pthreads over rows"}


def reference_arm(args, rank, world):
    cfg = W.config(args.config)
    if rank != 0:
        return None
    import oracle
    t, m, n, nt = oracle_sample(cfg, target_s=1.5)
    rng = np.random.Generator(np.random.PCG64(2))
    times = []
    for s in range(args.warmup + args.steps):
        rows = rng.integers(0, cfg.BH * cfg.S, size=n)
        t0 = time.perf_counter()
        oracle.attention_rows(t.q64, t.k64, t.v64, cfg.scale, rows, m)
        if s >= args.warmup:
            times.append(time.perf_counter() - t0)
    frac = n / (cfg.BH * cfg.S)
    sec = statistics.mean(times)
    v = frac / sec
    return {"metric": METRIC, "value": round(v, 6), "unit": "layers/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(sec * 1e3, 3), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": describe(cfg), "B": cfg.B, "H": cfg.H, "S": cfg.S, "D": cfg.D},
            "cpu_baseline": {"value": round(v, 6), "unit": "layers/s", "cores": nt, "kind": "oracle",
                             "sample": f"{n} random query rows per step ({frac:.4%} of one layer)"},
            "e2e": {"value": round(v, 6), "unit": "layers/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", type=int, default=2, help="BASELINE.json config index (1-5); default configs[1]")
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--tile-n", type=int, default=0, help="LS sub-vector width T (0 = library default)")
    ap.add_argument("--no-all-configs", dest="all_configs", action="store_false")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        res = reference_arm(args, rank, world)
        if res is not None:
            print(json.dumps(res), flush=True)
        return
    import torch
    if world > 1:
        torch.cuda.set_device(local_rank)
        torch.distributed.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    res = gpu_arm(args, rank, world, local_rank)
    if res is not None:
        if world == 1:
            res["cpu_baseline"] = cpu_baseline(W.config(args.config), args.cpu_seconds)
        print(json.dumps(res), flush=True)
    if world > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
