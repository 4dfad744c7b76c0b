"""Energy per layer under sustained load (diagnostic for the power-capped headline).

For each path: a CUDA graph of K back-to-back layer calls over rotating input sets is replayed for
`--preload` seconds (the 1 kW cap engages), then for `--seconds` more while NVML's total-energy
counter and the SM clock are read; energy/layer = dE / layers, time/layer from CUDA events.
A plain device copy moving the same number of DRAM bytes as the recomposed layer's ncu count is
measured the same way, to separate DRAM energy from SM-side energy.

    python tools/energy_ab.py [--config 3] [--paths default,unfused,two_kernels,copy]
"""
import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import pynvml  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_iiswc_choilkha22_b200 as sr  # noqa: E402
import workloads as W  # noqa: E402


def measure(fn_graph, K, preload, seconds, h):
    g = fn_graph
    t_end = time.perf_counter() + preload
    while time.perf_counter() < t_end:
        g.replay()
    torch.cuda.synchronize()
    clk, pw, stop = [], [], [False]

    def sampler():
        while not stop[0]:
            clk.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
            pw.append(pynvml.nvmlDeviceGetPowerUsage(h) / 1e3)
            time.sleep(0.02)

    th = threading.Thread(target=sampler)
    th.start()
    g.replay()  # warm, then the measured region
    torch.cuda.synchronize()
    e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    n = 0
    a.record()
    t_end = time.perf_counter() + seconds
    while time.perf_counter() < t_end:
        g.replay()
        n += K
    b.record()
    torch.cuda.synchronize()
    e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(h)
    stop[0] = True
    th.join()
    ms = a.elapsed_time(b)
    return {"us_per_layer": round(ms * 1e3 / n, 2), "mJ_per_layer": round((e1 - e0) / n, 3),
            "avg_W": round((e1 - e0) / ms, 1), "sm_mhz_median": statistics.median(clk) if clk else None,
            "power_w_median": round(statistics.median(pw), 1) if pw else None, "layers": n}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=3)
    ap.add_argument("--paths", default="default,unfused,two_kernels,copy")
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--preload", type=float, default=1.5)
    ap.add_argument("--seconds", type=float, default=1.5)
    args = ap.parse_args()
    pynvml.nvmlInit()
    vis = os.environ.get("CUDA_VISIBLE_DEVICES")
    h = pynvml.nvmlDeviceGetHandleByIndex(int(vis.split(",")[0]) if vis else 0)
    dev = torch.device("cuda", 0)
    cfg = W.config(args.config)
    L = bench.Layer(cfg, dev, seed_base=cfg.idx, sr=sr, torch=torch, variants=True)
    L.run()
    sets, _ = bench.rotation_sets(cfg, dev, 0, sr, torch, L, 0, None, variants=True)
    K = args.steps
    out = {"config": bench.describe(cfg)}
    ncu = bench.load_ncu_traffic().get(f"C{cfg.idx}", {})
    for p in args.paths.split(","):
        if p == "copy":
            nbytes = ncu.get("recomposed_dram_bytes") or 700_000_000
            bufs = [(torch.empty(nbytes // 2, dtype=torch.uint8, device=dev),
                     torch.empty(nbytes // 2, dtype=torch.uint8, device=dev)) for _ in range(2)]
            fns = [(lambda s=s: s[1].copy_(s[0])) for s in bufs]
        else:
            kw = {"default": {}, "unfused": {"fused": False}, "two_kernels": {"two_kernels": True},
                  "ir_kernel": {"ir_kernel": True}, "fuse_ir": {"fuse_ir": True}}[p]
            fns = [(lambda x=x, kw=kw: x.run(**kw)) for x in sets]
        g = bench.steps_graph(torch, fns, K)
        out[p] = measure(g, K, args.preload, args.seconds, h)
        if p == "copy":
            out[p]["bytes"] = nbytes
        print(p, out[p], flush=True)
        del g
        torch.cuda.empty_cache()
    print(json.dumps(out))


if __name__ == "__main__":
    main()
