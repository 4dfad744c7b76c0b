#!/usr/bin/env python
"""bench.py -- attention layers/s and HBM bytes/layer of the softmax-recomposed path vs the in-repo
unfused path on B200 (BASELINE.json "metric").

One step = one attention layer (all B*H heads of the workload config) through the C ABI's default
path: GEMM1 + Local Softmax (+ the IR merge inside GEMM1) -> GS + GEMM2.
Headline workload: C3 GPT-Neo (B4 H16 S2048 D128 bf16, causal), the largest BASELINE config, whose
285 MB attention matrix cannot stay on chip (the paper's premise).

Timing: inputs resident in HBM; K back-to-back layer calls (captured in one CUDA graph) cycling
through enough independent input/workspace sets that no step finds its data in L2; W untimed
warm-up steps; ONE timed region of exactly K steps between CUDA events on the launching stream,
barrier + synchronize on both sides, max over ranks.  Extra regions give the min/median/max spread.

Multi-GPU (torchrun, N ranks): the layer's B*H heads are split across the ranks (shard.py: contiguous,
cost-balanced head ranges; heads are independent, so no collective on the data
path); layer time = max over ranks of each rank's device time -> "scaling": "strong".  Each rank
running a full layer on its own inputs is reported beside it ("weak").

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 3] [--impl ours|reference]

--impl reference times the fp64 CPU oracle (this paper-only task's reference arm) on a bounded
sample of rows of the same workload, rank 0 only.
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
SPIN_CYCLES = 400_000  # ~0.2 ms at 1.97 GHz: device-side head start for the host enqueue
L2_BYTES = 126 << 20
NOMINAL_HBM_GBS = 8000.0  # the north star's "8 TB/s HBM roofline" (B200 DGX figure)
PAPER_CONTEXT = ("PAPER.md L9, L215: softmax recomposition gave 1.25x-1.65x end-to-end inference speedups on an "
                 "NVIDIA A100 over the same models without it (full models, real datasets) -- another GPU and another "
                 "metric; quoted as context, not a target")


def describe(cfg):
    m = {"dense": (("padding kv_len=" + str(cfg.kv_len)) if cfg.kv_len else ("causal" if cfg.causal else "none")),
         "blocksparse": "BigBird block 64: 3 window + 2 global + 3 random (622 blocks/head)",
         "window": f"sliding window {cfg.window} + {cfg.n_global} global" + (", causal" if cfg.causal else "")}[cfg.kind]
    return f"C{cfg.idx} {cfg.name}: B={cfg.B} H={cfg.H} S={cfg.S} D={cfg.D} {cfg.dtype}, mask: {m}"


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
        pw = [float(r[3]) for r in rows if r[3].strip().replace(".", "").isdigit()]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows), "power_w_median": statistics.median(pw) if pw else None}


def nvml_energy_reader(phys):
    """Callable returning the GPU's total energy counter in mJ (NVML), or None if unavailable."""
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(int(phys))
        pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
        return lambda: pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    except Exception:  # noqa: BLE001 -- no NVML / no counter: the energy fields are omitted
        return None


def sustained_energy(torch, g, K, seconds, read):
    """Replay the K-step graph back to back for `seconds`; (mJ per layer, ms per layer, layers)."""
    torch.cuda.synchronize()
    e0 = read()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record()
    n, t_end = 0, time.perf_counter() + seconds
    while time.perf_counter() < t_end:
        g.replay()
        n += K
    b.record()
    torch.cuda.synchronize()
    e1 = read()
    return (e1 - e0) / n, a.elapsed_time(b) / n, n


# ----------------------------------------------------------------------------- byte model

def alg_bytes(cfg, stored, T, BH=None):
    """Algorithmic HBM bytes per layer of the paper's three-kernel layout
    (SR_IR_KERNEL) and of the unfused path: Q, K, V, O once; the attention matrix written and read
    once (recomposed) or four times (unfused); m', d' written, read by IR, r'
    written and read."""
    e = 4 if cfg.dtype == "f32" else 2
    bhsd = (BH or cfg.BH) * cfg.S * cfg.D
    xe = 4 if cfg.dtype == "f32" else 2
    rows_tiles = stored / T  # (row, tile) pairs
    rec = {"gemm1_ls": 2 * bhsd * e + xe * stored + 8 * rows_tiles,
           "ir": 12 * rows_tiles,
           "gs_gemm2": xe * stored + 4 * rows_tiles + 2 * bhsd * e}
    unf = {"gemm1": 2 * bhsd * e + 2 * stored, "softmax": 4 * stored, "gemm2": 2 * stored + 2 * bhsd * e}
    return rec, unf


def alg_bytes_default(cfg, stored, T, BH=None):
    """Default path (IR merged in GEMM1): GEMM1 writes X' and m' (no d'), plus two partial (m, d) per
    query row; GEMM2 reads X', m' and the row statistics -- no IR kernel, no r'."""
    e = 4 if cfg.dtype == "f32" else 2
    bh = BH or cfg.BH
    bhsd = bh * cfg.S * cfg.D
    rows_tiles = stored / T
    rows = bh * cfg.S
    return {"gemm1_ls_ir": 2 * bhsd * e + 2 * stored + 4 * rows_tiles + 16 * rows,
            "gs_gemm2": 2 * stored + 4 * rows_tiles + 16 * rows + 2 * bhsd * e}


def alg_bytes_bwd(cfg, stored, T):
    """Training backward (NEXT-4), algorithmic HBM bytes per kernel."""
    e = 2
    bhsd = cfg.BH * cfg.S * cfg.D
    rt = stored / T
    rows = cfg.BH * cfg.S
    return {"prep": 2 * bhsd * e + 28 * rows,
            "ds": 4 * bhsd * e + 2 * stored + 4 * rt + 12 * rows + 2 * stored + 4 * rt,
            "dk": 2 * stored + 2 * bhsd * e,
            "dv": 2 * stored + 4 * rt + 2 * bhsd * e}


def flops(cfg, stored):
    return 4.0 * cfg.D * stored  # two GEMMs, 2 flops per MAC, over stored score elements


# ----------------------------------------------------------------------------- one layer (or one shard of it)

class Layer:
    """q, k, v, out, masks and workspaces of one layer of `cfg` -- or, with `shard`, of the heads
    [shard.g0, shard.g1) of that layer, re-packed as a layer of its own (shard.py)."""

    def __init__(self, cfg, device, seed_base, sr, torch, tile_n=0, shard=None, variants=True):
        from paper_conf_iiswc_choilkha22_b200 import shard as SH
        self.cfg, self.sr, self.torch, self.tile_n, self.shard = cfg, sr, torch, tile_n, shard
        t = W.make_qkv(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=seed_base)
        self.B, self.H = (cfg.B, cfg.H) if shard is None else shard.BH
        self.BH = self.B * self.H
        self.host, self.dev = {}, {}
        for n in ("q", "k", "v"):
            a = getattr(t, n + "_s")
            if cfg.dtype == "bf16":
                ht = torch.from_numpy(a.view(np.int16).copy()).view(torch.bfloat16)
            else:
                ht = torch.from_numpy(np.ascontiguousarray(a))
            if shard is not None:
                ht = SH.shard_view(ht, shard).contiguous()
            self.host[n] = ht.pin_memory()
            self.dev[n] = self.host[n].to(device)
        self.tdt = {"f32": torch.float32, "f16": torch.float16, "bf16": torch.bfloat16}[cfg.dtype]
        self.out = torch.empty((self.B, self.H, cfg.S, cfg.D), dtype=self.tdt, device=device)
        self.out_host = torch.empty_like(self.out, device="cpu").pin_memory()
        if cfg.kind == "dense":
            kv = cfg.kv_len if shard is None else shard.kv_len
            self.mask = sr.dense_mask(kv)
        elif cfg.kind == "blocksparse":
            self.mask = sr.block_mask(W.config_layout(cfg) if shard is None else shard.layout)
        else:
            self.mask = sr.window_mask(cfg.window, cfg.n_global)
        self.kw = dict(scale=cfg.scale, causal=cfg.causal)
        self.in_dt = sr.dtype_code(self.tdt)
        self.device = device

        def ws_for(**kw):
            info = sr.workspace_info(self.mask, self.B, self.H, cfg.S, cfg.D, self.in_dt, causal=cfg.causal, **kw)
            return torch.empty(info["total_bytes"], dtype=torch.uint8, device=device), info["tile_n"]

        self.ws = {}
        self.ws[True], self.T = ws_for(tile_n=tile_n)  # default path (16-bit: one launch, T = 64)
        self.n_tiles, self.stored = self.stats(self.T)
        if cfg.dtype != "f32":
            self.ws[False], self.Tu = ws_for(fused=False, tile_n=64)  # unfused at the default path's T
            self.stored_u = self.stats(64)[1]
            if variants:
                # two-launch variants (SR_TWO_KERNELS, SR_FUSE_IR, SR_IR_KERNEL) at their tuned T (128; 64
                # for block-sparse), the unfused baseline also at T = 128, SD at its library default
                self.T2 = 64 if cfg.kind == "blocksparse" else 128
                self.ws["t2"], _ = ws_for(tile_n=self.T2)
                self.stored2 = self.stats(self.T2)[1]
                self.ws["u128"], _ = ws_for(fused=False, tile_n=self.T2)
                self.ws["sd"], self.Tsd = ws_for(sd=True)

    def stats(self, T):
        return self.sr.schedule_stats(self.mask, self.B, self.H, self.cfg.S, causal=self.cfg.causal, tile_n=T)

    def setup_train(self, seed_base):
        """Training (NEXT-4): dE/dO, gradient buffers and an SR_WS_TRAIN workspace."""
        cfg, torch, sr = self.cfg, self.torch, self.sr
        do_s, _ = W.make_dout(cfg.B, cfg.H, cfg.S, cfg.D, cfg.dtype, seed_base=seed_base)
        if cfg.dtype == "bf16":
            self.dout = torch.from_numpy(do_s.view(np.int16).copy()).view(torch.bfloat16).to(self.out.device)
        else:
            self.dout = torch.from_numpy(np.ascontiguousarray(do_s)).to(self.out.device)
        info = sr.workspace_info(self.mask, self.B, self.H, cfg.S, cfg.D, sr.dtype_code(self.dout.dtype),
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
                                dq=dq, dk=dk, dv=dv, stages=stages, tile_n=self.tile_n,
                                sched_resident=stages != 0, **self.kw)

    def train_step(self):
        self.fwd_train()
        self.bwd()

    def run(self, fused=True, stages=0, q=None, k=None, v=None, fuse_ir=False, sd=False, ir_kernel=False,
            two_kernels=False, unfused_T=64, resident=False, concurrent=False, gs_prologue=False):
        d = self.dev
        two = fuse_ir or ir_kernel or two_kernels
        if sd:
            ws, tn = self.ws["sd"], 0
        elif not fused:
            ws, tn = (self.ws[False], 64) if unfused_T == 64 else (self.ws["u128"], self.T2)
        elif two:
            ws, tn = self.ws["t2"], self.T2
        else:
            ws, tn = self.ws[True], self.tile_n
        return self.sr.call(self.mask, q if q is not None else d["q"], k if k is not None else d["k"],
                            v if v is not None else d["v"], out=self.out, fused=fused, stages=stages,
                            workspace=ws, tile_n=tn, fuse_ir=fuse_ir, sd=sd, ir_kernel=ir_kernel,
                            two_kernels=two_kernels, concurrent=concurrent, gs_prologue=gs_prologue,
                            # single-kernel timing: the schedule is already in the workspace
                            sched_resident=resident or stages != 0, **self.kw)


# ----------------------------------------------------------------------------- timing helpers

def timed(torch, fn, steps, warmup, flush):
    """W warm-up + K timed single calls; L2 flushed before each; returns per-call device ms list."""
    ev = []
    for s in range(warmup + steps):
        if flush is not None:
            flush[0].zero_()  # write 256 MiB (evicts everything) ...
            flush[1].sum()  # ... then read another 256 MiB so L2 starts the step clean, not dirty
        # keep the GPU busy (outside the timed region) while the host enqueues the step
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


def rotation_sets(cfg, device, rank, sr, torch, L, tile_n, shard=None, variants=True):
    """Independent (q, k, v, out, workspace) sets for back-to-back timing: enough of them that the
    data cycled through between two uses of a set exceeds 2x the L2, so no step finds its inputs or
    its X' in L2 (the 'inputs larger than L2' form of the no-warm-cache rule)."""
    per = sum(t.numel() * t.element_size() for t in (L.dev["q"], L.dev["k"], L.dev["v"], L.out)) + L.ws[True].numel()
    n = max(2, min(8, math.ceil(2 * L2_BYTES / per)))
    sets = [L] + [Layer(cfg, device, seed_base=cfg.idx + 1000 * rank + 100 * i, sr=sr, torch=torch, tile_n=tile_n,
                        shard=shard, variants=variants) for i in range(1, n)]
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


def region(torch, g, K, spin=SPIN_CYCLES, warm=None):
    """Device ms per layer of one replay of the K-step graph (events around it).  Before the first
    event the device either spins (so a late host submission of the replay never shows up as idle
    time inside the region) or, with `warm`, runs that graph once more untimed: the timed steps then
    start from the steady state of the preceding warm-up steps (a region that starts cold, right
    after the idle sync, runs slower under the 1 kW power cap while the clock controller reacts)."""
    if warm is not None:
        warm.replay()
    else:
        torch.cuda._sleep(spin)
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record()
    g.replay()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / K


def sustained_regions(torch, g, K, n, preload_s, min_replays=1):
    """Replays of the K-step graph enqueued for `preload_s` seconds with no synchronisation, then n
    event-timed regions of one replay each, back to back, one synchronize at the end: the regions run
    in the power state the preceding load settled into, with no idle gap in which the clock can
    boost.  Device ms per step of each region."""
    t_end = time.perf_counter() + preload_s
    done = 0
    while done < min_replays or time.perf_counter() < t_end:
        g.replay()
        done += 1
    evs = []
    for _ in range(n):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        evs.append((a, b))
    torch.cuda.synchronize()
    return [a.elapsed_time(b) / K for a, b in evs]


def back_to_back(torch, fns, K, W_, reps=3):
    """Warm-up replays covering >= W_ steps, then `reps` timed regions of K steps; per-step ms list."""
    g = steps_graph(torch, fns, K)
    for _ in range(max(1, -(-W_ // K))):
        g.replay()
    torch.cuda.synchronize()
    return [region(torch, g, K) for _ in range(reps)]


def spread(xs):
    return {"min": round(min(xs), 5), "median": round(statistics.median(xs), 5), "max": round(max(xs), 5),
            "n_regions": len(xs)}


def capture(torch, fn):
    """CUDA graph of one call of fn (calls are capturable: include/sr_mha.h Ownership)."""
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


def make_shard(cfg, rank, world, T=64):
    from paper_conf_iiswc_choilkha22_b200 import shard as SH
    return SH.make_shard(rank, world, cfg.B, cfg.H, cfg.S, kv_len=cfg.kv_len, layout=W.config_layout(cfg), T=T,
                         causal=cfg.causal, kind=cfg.kind, window=cfg.window, n_global=cfg.n_global)


# ----------------------------------------------------------------------------- GPU arm

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
    tc_peak = peaks.get("bf16_tflops", 1590.0)
    cfg = W.config(args.config)
    f32 = cfg.dtype == "f32"
    flush = None if args.no_flush else (torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=device),
                                        torch.ones(FLUSH_BYTES // 4, dtype=torch.float32, device=device))
    shard = make_shard(cfg, rank, world) if world > 1 else None
    L = Layer(cfg, device, seed_base=cfg.idx, sr=sr, torch=torch, tile_n=args.tile_n, shard=shard,
              variants=world == 1)
    K, Wm = args.steps, args.warmup

    # ---- headline: K back-to-back layers (this rank's heads of ONE layer), one timed region
    L.run()
    n0 = sr.launch_count()
    L.run()
    launches_per_layer = sr.launch_count() - n0
    sets, rot_bytes = rotation_sets(cfg, device, rank, sr, torch, L, args.tile_n, shard, variants=False)
    n_sets = len(sets)
    g_tp = steps_graph(torch, [x.run for x in sets], K)
    for _ in range(max(1, -(-Wm // K))):  # >= W untimed warm-up steps
        g_tp.replay()
    # the same region on a GPU that was idle (boost clock, before the power cap engages): `burst`
    barrier(torch, world)
    ms_burst = dist_max(torch, region(torch, g_tp, K, warm=g_tp), world)
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    phys = vis.split(",")[local_rank] if vis else str(local_rank)
    clk = Clocks(phys)
    clk.start()
    energy_read = nvml_energy_reader(phys)
    energy = None
    if energy_read is not None:  # keep the GPU under this load (0.8 s) while nvidia-smi samples
        mj, ms_sus, n_sus = sustained_energy(torch, g_tp, K, 0.8, energy_read)
        energy = {"recomposed_mJ_per_layer": round(mj, 3), "recomposed_ms_per_layer": round(ms_sus, 5),
                  "layers": n_sus}
    else:
        t_end = time.perf_counter() + 0.8
        while time.perf_counter() < t_end:
            g_tp.replay()
    torch.cuda.synchronize()
    # the one-launch kernel alone (schedule resident: no upload launch), for the roofline's kernel
    # duration; its graph is built now, so no capture (and its idle gaps) falls between the timed regions
    g_res = steps_graph(torch, [(lambda x=x: x.run(resident=True)) for x in sets], K) if not f32 else None
    barrier(torch, world)
    # THE timed region: exactly K steps, after >= W untimed warm-up steps on the same stream -- 0.3 s of
    # replays of the same K-step graph enqueued with no synchronisation, so the region starts in the
    # sustained (power-capped) state instead of on a clock that boosted during an idle gap -- then the
    # region and 4 more, back to back; barrier + synchronize before the warm-up and after
    sus = sustained_regions(torch, g_tp, K, 5, 0.3, min_replays=-(-Wm // K))
    ms_rank, extra = sus[0], sus[1:]
    barrier(torch, world)
    # the kernel alone in the same state, right after (0.1 s of its own replays first)
    ms_res = sustained_regions(torch, g_res, K, 3, 0.1) if g_res is not None else None
    clocks = clk.stop()
    ms_step = dist_max(torch, ms_rank, world)
    step_spread = spread([dist_max(torch, x, world) for x in [ms_rank] + extra])
    launches = launches_per_layer * K

    # ---- the dominant kernel: the one-launch kernel (tc_fused) timed alone, back to back, with its
    # schedule already resident (isolates it from a schedule-upload launch when the schedule does not
    # fit the kernel's parameters; equal to the step when it does)
    if f32:
        kern = {}
        hb = alg_bytes(cfg, L.stored, L.T, BH=L.BH)[0]
        for name, bit in (("gemm1_ls", 1), ("ir", 2), ("gs_gemm2", 4)):
            t = statistics.mean(timed(torch, lambda b=bit: L.run(stages=b), K, Wm, flush))
            kern[name] = {"us": round(t * 1e3, 3), "alg_bytes": int(hb[name]), "GB/s": round(hb[name] / (t * 1e-3) / 1e9, 1)}
        dom = max(kern, key=lambda n: kern[n]["us"])
        dom_us = kern[dom]["us"]
        dom_bytes = kern[dom]["alg_bytes"]
        layer_bytes = sum(hb.values())
    else:
        hb = alg_bytes_default(cfg, L.stored, L.T, BH=L.BH)
        layer_bytes = sum(hb.values())
        dom, dom_us, dom_bytes = "sr_layer_one_kernel", statistics.median(ms_res) * 1e3, layer_bytes
        kern = {dom: {"us": round(dom_us, 3), "alg_bytes": int(dom_bytes), "GB/s": round(dom_bytes / (dom_us * 1e-6) / 1e9, 1),
                      "how": "median of 3 back-to-back regions of K calls with the schedule resident (no upload "
                             "launch), timed right after the headline regions, same power state",
                      "share_of_step": round(dom_us * 1e-3 / ms_step, 4)}}
    ms_kern = dist_max(torch, dom_us * 1e-3, world)

    # ---- unfused in-repo baseline (same tiles, same skipping), at the default path's T = 64
    unf = None
    if not f32:
        ub = alg_bytes(cfg, L.stored_u, 64, BH=L.BH)[1]
        ms_unf = dist_max(torch, statistics.median(
            back_to_back(torch, [(lambda x=x: x.run(fused=False)) for x in sets], K, Wm)), world)
        if energy is not None and world == 1:  # the unfused layer's board energy under the same sustained load
            g_un = steps_graph(torch, [(lambda x=x: x.run(fused=False)) for x in sets], K)
            mj_u, ms_u, n_u = sustained_energy(torch, g_un, K, 0.8, energy_read)
            del g_un
            energy.update({"unfused_mJ_per_layer": round(mj_u, 3), "unfused_ms_per_layer": round(ms_u, 5),
                           "reduction": round(1 - energy["recomposed_mJ_per_layer"] / mj_u, 4),
                           "how": "NVML total-energy counter (whole board) over 0.8 s of back-to-back layers "
                                  "of each path (the K-step graph replayed), divided by the layers run; the "
                                  "paper's claim is a 29 % cut of off-chip access energy (PAPER.md L27)"})
        unf = {"value": round(1e3 / ms_unf, 2), "ms_per_step": round(ms_unf, 5), "T": 64,
               "alg_bytes": int(sum(ub.values())),
               "speedup_recomposed_vs_unfused": round(ms_unf / ms_step, 3),
               "byte_reduction_alg": round(1 - layer_bytes / sum(ub.values()), 4)}
        if world == 1:
            kern_unf = {}
            for name, bit in (("gemm1", 1), ("softmax", 2), ("gemm2", 4)):
                # back to back over the rotating sets (the layer's own measurement method: no launch /
                # event floor per call, no set's data left in L2), and a single L2-flushed call beside it
                t = statistics.median(back_to_back(torch, [(lambda x=x, b=bit: x.run(fused=False, stages=b))
                                                           for x in sets], K, Wm))
                t1 = statistics.mean(timed(torch, lambda b=bit: L.run(fused=False, stages=b), K, Wm, flush))
                kern_unf[name] = {"us": round(t * 1e3, 3), "alg_bytes": int(ub[name]),
                                  "GB/s": round(ub[name] / (t * 1e-3) / 1e9, 1),
                                  "frac": round(ub[name] / (t * 1e-3) / 1e9 / hbm_peak, 4),
                                  "us_single_call_l2_flushed": round(t1 * 1e3, 3)}
            unf["kernels"] = kern_unf
            unf["kernels_how"] = ("per stage: K back-to-back stage-only calls over the rotating input/workspace "
                                  "sets (schedule resident), median of 3 regions; us_single_call_l2_flushed: one "
                                  "call between events after a 256 MiB L2 flush")
            ub2 = alg_bytes(cfg, L.stored2, L.T2)[1]
            ms_u2 = statistics.median(back_to_back(torch, [lambda: L.run(fused=False, unfused_T=L.T2)], K, Wm))
            unf["at_T%d" % L.T2] = {"ms_per_step": round(ms_u2, 5), "alg_bytes": int(sum(ub2.values())),
                                    "note": "same baseline at T = %d (one input set: L2-warm inputs)" % L.T2}

    # ---- variants: two launches, IR in GEMM2, the paper's standalone IR kernel, SD (N = 1)
    variants = None
    if not f32 and world == 1:
        def graph_ms(**kw):
            g = capture(torch, lambda: L.run(**kw))
            return statistics.mean(timed(torch, g.replay, K, Wm, flush))

        def stage_us(bit, **kw):
            L.run(**kw)
            return statistics.mean(timed(torch, lambda: L.run(stages=bit, **kw), K, Wm, flush)) * 1e3

        def kd(times, nbytes):
            return {n: {"us": round(t, 3), "alg_bytes": int(nbytes[n]), "GB/s": round(nbytes[n] / (t * 1e-6) / 1e9, 1),
                        "frac": round(nbytes[n] / (t * 1e-6) / 1e9 / hbm_peak, 4)} for n, t in times.items()}

        b2 = alg_bytes_default(cfg, L.stored2, L.T2)
        r2 = alg_bytes(cfg, L.stored2, L.T2)[0]
        rt2 = L.stored2 / L.T2
        ms_two, ms_fir, ms_irk, ms_sd = (graph_ms(two_kernels=True), graph_ms(fuse_ir=True),
                                         graph_ms(ir_kernel=True), graph_ms(sd=True))
        kern_two = {n: stage_us(bit, two_kernels=True) for n, bit in (("gemm1_ls_ir", 1), ("gs_gemm2", 4))}
        kern_irk = {n: stage_us(bit, ir_kernel=True) for n, bit in (("gemm1_ls", 1), ("ir", 2), ("gs_gemm2", 4))}
        irk_share = kern_irk["ir"] / sum(kern_irk.values())
        # the IR kernel back to back (K launches in one graph, PDL-chained): its launch-to-launch time
        # without the ~6 us single-launch event floor (diagnostic: its 8-23 MB of statistics stay L2-warm)
        ir_b2b = statistics.median(back_to_back(torch, [lambda: L.run(ir_kernel=True, stages=2)], K, Wm)) * 1e3
        variants = {
            "how": "single-call CUDA-graph replays, L2 flushed before each; kernels: stage-selected launches",
            "two_kernels": {"what": f"GEMM1+LS+IR -> GS+GEMM2 as two launches (SR_TWO_KERNELS, T={L.T2})",
                            "ms_per_step": round(ms_two, 5), "alg_bytes": int(sum(b2.values())), "kernels": kd(kern_two, b2)},
            "fused_ir": {"what": f"IR folded into GS+GEMM2 (SURVEY NEXT-2, 2 kernels, T={L.T2})",
                         "ms_per_step": round(ms_fir, 5), "alg_bytes": int(sum(r2.values()) - 4 * rt2)},
            "ir_kernel": {"what": "the paper's three-kernel layout: GEMM1+LS -> standalone IR kernel (writes r') -> "
                                  f"GS+GEMM2 (SR_IR_KERNEL, PAPER.md L165-L173, T={L.T2})",
                          "ms_per_step": round(ms_irk, 5), "alg_bytes": int(sum(r2.values())),
                          "kernels": kd(kern_irk, r2), "ir_share_of_layer": round(irk_share, 4),
                          "ir_back_to_back": {"us": round(ir_b2b, 3), "GB/s": round(r2["ir"] / (ir_b2b * 1e-6) / 1e9, 1),
                                              "frac": round(r2["ir"] / (ir_b2b * 1e-6) / 1e9 / hbm_peak, 4),
                                              "share_of_layer": round(ir_b2b * 1e-3 / ms_irk, 4),
                                              "note": "L2-warm statistics; diagnostic, not a roofline claim"}},
            "sd": {"what": f"decomposition without fusion: GEMM1 -> LS -> IR -> GS -> GEMM2 (PAPER.md SD, NEXT-1, T={L.Tsd})",
                   "ms_per_step": round(ms_sd, 5)}}
        L.run()

    # ---- training: forward + backward of the layer on one SR_WS_TRAIN workspace
    train = None
    if not f32 and world == 1:
        L.setup_train(cfg.idx)
        L.train_step()
        g_tr = capture(torch, L.train_step)
        ms_tr = statistics.mean(timed(torch, g_tr.replay, K, Wm, flush))
        g_bw = capture(torch, L.bwd)
        ms_bw = statistics.mean(timed(torch, g_bw.replay, K, Wm, flush))
        bb = alg_bytes_bwd(cfg, L.stored, L.T)
        kern_bw = {}
        for name, bit, keys in (("prep_ds_dq", 1, ("prep", "ds")), ("dk_dv", 4, ("dk", "dv"))):
            t = statistics.mean(timed(torch, lambda b=bit: L.bwd(stages=b), K, Wm, flush))
            nb = sum(bb[k_] for k_ in keys)
            kern_bw[name] = {"us": round(t * 1e3, 3), "alg_bytes": int(nb), "GB/s": round(nb / (t * 1e-3) / 1e9, 1)}
        train = {"what": "forward (default path) + backward (sr_mha_*_bwd; Eq. 3 with y = X' r' recomposed per tile); "
                         "single-call CUDA-graph replays, L2 flushed before each",
                 "fwd_bwd_ms": round(ms_tr, 5), "bwd_ms": round(ms_bw, 5), "alg_bytes_bwd": int(sum(bb.values())),
                 "bwd_hbm_GBps": round(sum(bb.values()) / (ms_bw * 1e-3) / 1e9, 1), "kernels": kern_bw}

    # ---- end to end through the public API: pinned host -> device, layer, device -> host
    h2d = sum(L.host[n].numel() * L.host[n].element_size() for n in ("q", "k", "v"))
    d2h = L.out.numel() * L.out.element_size()
    barrier(torch, world)
    ms_e2e, e2e_same = e2e_pipelined(torch, L, K, Wm)
    ms_e2e = dist_max(torch, ms_e2e, world)

    # ---- weak scaling (N > 1): every rank runs the FULL layer on its own inputs
    weak = None
    if world > 1:
        del sets, g_tp
        torch.cuda.empty_cache()
        Lf = Layer(cfg, device, seed_base=cfg.idx + 1000 * rank, sr=sr, torch=torch, tile_n=args.tile_n, variants=False)
        sets_f, _ = rotation_sets(cfg, device, rank, sr, torch, Lf, args.tile_n, None, variants=False)
        barrier(torch, world)
        ms_w = dist_max(torch, statistics.median(back_to_back(torch, [x.run for x in sets_f], K, Wm)), world)
        weak = {"value": round(world * 1e3 / ms_w, 2), "ms_per_step": round(ms_w, 5),
                "what": "each rank runs its own full layer (per-GPU work fixed as N grows)"}
        del Lf, sets_f

    # ---- N = 1: the head-sharded layer's per-rank time at k = 2, 4, 8, each shard measured here
    strong_model = None
    if world == 1 and args.shard_model:
        del sets, g_tp
        torch.cuda.empty_cache()
        strong_model = shard_model(args, cfg, device, sr, torch, K, Wm, ms_step)

    # ---- NEXT-3 (Fig. 9): sequence length and batch around GPT-Neo (C3), N = 1
    sweep = None
    if world == 1 and args.sweep and cfg.idx == 3:
        sweep = sweep_points(cfg, device, sr, torch, hbm_peak)

    # ---- other configs (same run): layers/s and bytes, recomposed vs unfused, with spread
    others = {}
    if args.all_configs and world == 1:
        for c2 in W.CONFIGS + W.EXTRA_CONFIGS:
            if c2.idx == cfg.idx:
                continue
            others[f"C{c2.idx}"] = other_config(c2, device, sr, torch, hbm_peak)
            torch.cuda.empty_cache()

    if rank != 0:
        return None
    ncu = load_ncu_traffic().get(f"C{cfg.idx}", {})
    achieved = dom_bytes / (ms_kern * 1e-3) / 1e9
    dram = ncu.get(f"{dom}_dram_bytes")
    value = 1e3 / ms_step
    res = {
        "metric": METRIC,
        "value": round(value, 2),
        "unit": "layers/s",
        "n_gpus": world, "steps": K, "warmup": Wm,
        "ms_per_step": round(ms_step, 5),
        "timing": f"one region of exactly K={K} back-to-back layer calls (C ABI, captured in one CUDA graph) between "
                  f"two events, right after >= W={Wm} untimed warm-up steps on the same stream (0.3 s of replays "
                  "enqueued with no synchronisation: the sustained, power-capped state), barrier + synchronize "
                  "before the warm-up and after the region, max over ranks; "
                  f"{n_sets} rotating input/workspace sets "
                  f"({rot_bytes / 2**20:.0f} MiB > 2x L2) so no step finds its data in L2; step_ms = spread over "
                  "that region and 4 more",
        "step_ms": step_spread,
        "burst": {"value": round(1e3 / ms_burst, 2), "ms_per_step": round(ms_burst, 5),
                  "what": "the same K-step region on a GPU coming out of idle (boost clock): the headline "
                          "`value` is the sustained one, timed after 0.8 s of this load, when the 1 kW power cap "
                          "(sw_power_cap in `clocks`) has lowered the SM clock"},
        "higher_is_better": True,
        "scaling": "strong" if world > 1 else "weak",
        "vs_baseline": None,
        "dtype": cfg.dtype,
        "data": "synthetic (seeded N(0,1) q/k/v rounded to dtype; no datasets or weights needed)",
        "config": {"workload": describe(cfg), "B": cfg.B, "H": cfg.H, "S": cfg.S, "D": cfg.D, "T": L.T,
                   "tiles": L.n_tiles, "stored_score_elems": L.stored,
                   "l2": "inputs larger than L2: rotating sets, >2x L2 cycled between uses of a set; single-call "
                         "timings flush L2 (256 MiB write + 256 MiB read) before each call",
                   "parallelism": (f"heads{world} (one layer's B*H heads split across {world} ranks, "
                                   f"this rank's heads {shard.g0}..{shard.g1 - 1})") if world > 1 else "1 GPU"},
        "hbm_bytes_per_layer": None if f32 else {
            "recomposed_alg": int(layer_bytes), "unfused_alg": unf["alg_bytes"],
            "reduction_alg": unf["byte_reduction_alg"],
            "recomposed_ncu_dram": ncu.get("recomposed_dram_bytes"), "unfused_ncu_dram": ncu.get("unfused_dram_bytes"),
            "reduction_ncu_dram": (round(1 - ncu["recomposed_dram_bytes"] / ncu["unfused_dram_bytes"], 4)
                                   if ncu.get("recomposed_dram_bytes") and ncu.get("unfused_dram_bytes") else None),
            "ncu_source": "profiles/ncu_traffic.json (ncu dram__bytes_read.sum + dram__bytes_write.sum per launch)"},
        "unfused": unf,
        "energy": energy,
        "variants": variants,
        "kernels": kern,
        "roofline": {"kernel": dom, "bound": "hbm", "achieved": round(achieved, 1), "peak": hbm_peak, "unit": "GB/s",
                     "frac": round(achieved / hbm_peak, 4), "traffic": dram, "peak_source": peak_src,
                     "achieved_how": "algorithmic bytes of the layer (DESIGN.md §6) / the kernel's duration",
                     "frac_of_nominal_8TBps": round(achieved / NOMINAL_HBM_GBS, 4),
                     "dram_frac": (round(dram / (ms_kern * 1e-3) / 1e9 / hbm_peak, 4) if dram else None),
                     "tensor_frac": round(flops(cfg, L.stored) / (ms_kern * 1e-3) / 1e12 / tc_peak, 4),
                     "burst": {"achieved": round(layer_bytes / (ms_burst * 1e-3) / 1e9, 1),
                               "frac": round(layer_bytes / (ms_burst * 1e-3) / 1e9 / hbm_peak, 4),
                               "what": "the same bytes over the burst step time (boost clock, before the power "
                                       "cap engages; the step is the kernel plus its schedule upload)"}},
        "e2e": {"value": round(1e3 / ms_e2e, 2), "unit": "layers/s", "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": int(d2h), "ms_per_step": round(ms_e2e, 5),
                "how": "K steps through the public API, each H2D of its q/k/v from pinned host memory, the "
                       "layer, D2H of its output; copy-in / compute / copy-out streams, double-buffered"
                       + ("; per rank: its shard's bytes" if world > 1 else ""),
                "output_bitwise_equal_device_path": bool(e2e_same),
                "pcie_GBps_per_gpu": round((h2d + d2h) / (ms_e2e * 1e-3) / 1e9, 1)},
        "gpu_launches": int(launches),
        "launches_per_layer": int(launches_per_layer),
        "training": train,
        "weak": weak,
        "strong_scaling_shards": strong_model,
        "sweep": sweep,
        "paper_context": PAPER_CONTEXT,
        "clocks": clocks,
    }
    if others:
        res["all_configs"] = others
    return res


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

    def go(n):
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

    go(max(warmup, nbuf))
    torch.cuda.synchronize()
    torch.cuda._sleep(SPIN_CYCLES)
    a, b = go(steps)
    torch.cuda.synchronize()
    # every step computed the same layer from the same host inputs: the pipelined result read back
    # to the host must equal the device path's output bit for bit (the kernels are deterministic)
    L.run()
    torch.cuda.synchronize()
    same = all(torch.equal(h, L.out.cpu()) for h in hosts)
    return a.elapsed_time(b) / steps, same


def shard_model(args, cfg, device, sr, torch, K, Wm, ms_full):
    """Strong scaling of the head-sharded layer, measured shard by shard on this one GPU: for k ranks,
    each rank's work is exactly its shard (no exchange step), so the layer time at k GPUs is the max
    over the k shard times.  Distinct shards only (identical head ranges cost the same)."""
    out = {"how": "each distinct shard of the k-way head split timed here as its own layer (back to back, "
                  "inputs larger than L2); layer time at k GPUs = max over shards", "k": {}}
    for k in (2, 4, 8):
        seen, worst, items = {}, 0.0, None
        for r in range(k):
            sh = make_shard(cfg, r, k)
            key = (sh.n, None if sh.kv_len is None else tuple(sh.kv_len.tolist()),
                   None if cfg.kind != "blocksparse" else (sh.g0 % cfg.H, sh.n))
            if key in seen:
                continue
            Ls = Layer(cfg, device, seed_base=cfg.idx, sr=sr, torch=torch, tile_n=args.tile_n, shard=sh, variants=False)
            sets, _ = rotation_sets(cfg, device, 0, sr, torch, Ls, args.tile_n, sh, variants=False)
            t = statistics.median(back_to_back(torch, [x.run for x in sets], K, Wm))
            seen[key] = t
            worst = max(worst, t)
            del Ls, sets
            torch.cuda.empty_cache()
        out["k"][str(k)] = {"layer_ms": round(worst, 5), "layers_per_s": round(1e3 / worst, 2),
                            "efficiency_vs_1gpu": round(ms_full / (k * worst), 4),
                            "distinct_shards": len(seen)}
    return out


def sweep_points(cfg, device, sr, torch, hbm_peak):
    """GPT-Neo attention at L = 512 .. 4096 (batch 4) and batch 1 .. 8 (L = 2048): layers/s of the
    default path and of the unfused baseline, back to back with inputs larger than L2 (
    parity of these shapes: tests/test_gpu_sweep.py)."""
    import dataclasses
    out = []
    for axis, S, B in [("L", 512, 4), ("L", 1024, 4), ("L", 2048, 4), ("L", 4096, 4),
                       ("batch", 2048, 1), ("batch", 2048, 2), ("batch", 2048, 8)]:
        c = dataclasses.replace(cfg, S=S, B=B, name=f"gptneo_L{S}_B{B}")
        Ls = Layer(c, device, seed_base=c.idx, sr=sr, torch=torch, variants=False)
        sets, _ = rotation_sets(c, device, 0, sr, torch, Ls, 0, None, variants=False)
        tr = statistics.median(back_to_back(torch, [x.run for x in sets], 10, 3, reps=3))
        tu = statistics.median(back_to_back(torch, [(lambda x=x: x.run(fused=False)) for x in sets], 10, 3, reps=3))
        rb = sum(alg_bytes_default(c, Ls.stored, Ls.T).values())
        out.append({"axis": axis, "L": S, "B": B, "layers_per_s": round(1e3 / tr, 1), "ms": round(tr, 5),
                    "unfused_ms": round(tu, 5), "speedup_vs_unfused": round(tu / tr, 3),
                    "roofline_frac": round(rb / (tr * 1e-3) / 1e9 / hbm_peak, 4)})
        del Ls, sets
        torch.cuda.empty_cache()
    return out


def other_config(c2, device, sr, torch, hbm_peak):
    L2 = Layer(c2, device, seed_base=c2.idx, sr=sr, torch=torch, variants=False)
    sets2, _ = rotation_sets(c2, device, 0, sr, torch, L2, 0, None, variants=False)
    tr_all = back_to_back(torch, [x.run for x in sets2], 10, 3, reps=5)
    tr = statistics.median(tr_all)
    ncu = load_ncu_traffic().get(f"C{c2.idx}", {})
    if c2.dtype == "f32":
        r2 = alg_bytes(c2, L2.stored, L2.T)[0]
        return {"workload": describe(c2), "layers_per_s": round(1e3 / tr, 1), "ms": round(tr, 5), "step_ms": spread(tr_all),
                "alg_bytes_recomposed": int(sum(r2.values())), "note": "fp32 SIMT path; launch-bound (4.2 MFLOP)"}
    r2 = alg_bytes_default(c2, L2.stored, L2.T)
    u2 = alg_bytes(c2, L2.stored_u, 64)[1]
    tu_all = back_to_back(torch, [(lambda x=x: x.run(fused=False)) for x in sets2], 10, 3, reps=5)
    tu = statistics.median(tu_all)
    ent = {"workload": describe(c2), "layers_per_s": round(1e3 / tr, 1), "ms": round(tr, 5), "step_ms": spread(tr_all),
           "alg_bytes_recomposed": int(sum(r2.values())), "unfused_ms": round(tu, 5), "unfused_step_ms": spread(tu_all),
           "alg_bytes_unfused": int(sum(u2.values())), "byte_reduction_alg": round(1 - sum(r2.values()) / sum(u2.values()), 4),
           "speedup_vs_unfused": round(tu / tr, 3),
           "roofline_frac": round(sum(r2.values()) / (tr * 1e-3) / 1e9 / hbm_peak, 4),
           "frac_of_nominal_8TBps": round(sum(r2.values()) / (tr * 1e-3) / 1e9 / NOMINAL_HBM_GBS, 4),
           "ncu_dram_bytes_recomposed": ncu.get("recomposed_dram_bytes"),
           "ncu_dram_bytes_unfused": ncu.get("unfused_dram_bytes")}
    ent["unfused_kernels"] = {}  # the baseline's own kernels, back to back (schedule resident)
    for name, bit in (("gemm1", 1), ("softmax", 2), ("gemm2", 4)):
        t = statistics.median(back_to_back(torch, [(lambda x=x, b=bit: x.run(fused=False, stages=b)) for x in sets2],
                                           10, 3))
        ent["unfused_kernels"][name] = {"us": round(t * 1e3, 3),
                                        "frac": round(u2[name] / (t * 1e-3) / 1e9 / hbm_peak, 4)}
    x_bytes = 2 * L2.stored
    if x_bytes < 0.5 * L2_BYTES:
        ent["note"] = (f"X' ({x_bytes / 1e6:.1f} MB) is L2-resident: the kernel reads it back from L2, so its DRAM "
                       "traffic is little more than Q, K, V, O -- roofline_frac is an effective rate, not DRAM throughput")
    del L2, sets2
    return ent


# ----------------------------------------------------------------------------- CPU (oracle) arm

def oracle_mask_for(cfg):
    import oracle
    if cfg.kind == "dense":
        return oracle.Mask(kv_len=cfg.kv_len, causal=cfg.causal)
    if cfg.kind == "blocksparse":
        return oracle.Mask(kind="block", layout=W.config_layout(cfg), causal=cfg.causal)
    return oracle.Mask(kind="window", window=cfg.window, n_global=cfg.n_global, causal=cfg.causal)


def oracle_sample(cfg, target_s, seed=0):
    """Size a bounded random sample of rows for ~target_s of fp64 oracle work; returns (tensors, mask, rows, threads)."""
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
            "warmup": args.warmup, "ms_per_step": round(sec * 1e3, 3), "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak",
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
    ap.add_argument("--config", type=int, default=3,
                    help="BASELINE.json config index (1-5; 6 = GPT-Neo local attention); default 3, the largest")
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--tile-n", type=int, default=0, help="LS sub-vector width T (0 = library default)")
    ap.add_argument("--no-all-configs", dest="all_configs", action="store_false")
    ap.add_argument("--no-shard-model", dest="shard_model", action="store_false")
    ap.add_argument("--no-sweep", dest="sweep", action="store_false")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    # SR_BENCH_SHARED_GPU=1: a functional check of the N > 1 code path on a one-GPU box -- every rank
    # on cuda:0, gloo for the host-side plumbing; the timings of such a run mean nothing
    shared = os.environ.get("SR_BENCH_SHARED_GPU") == "1"
    if shared:
        local_rank = 0
    if args.impl == "reference":
        res = reference_arm(args, rank, world)
        if res is not None:
            print(json.dumps(res), flush=True)
        return
    import torch
    if world > 1:
        torch.cuda.set_device(local_rank)
        if shared:
            torch.distributed.init_process_group("gloo")
        else:
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
