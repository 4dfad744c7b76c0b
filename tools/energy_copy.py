"""Board energy per DRAM byte (NVML): idle power, then back-to-back device copies (torch copy_ of
1 GiB bf16 buffers, read + write bytes) for ~1.5 s after a warm-up.  Diagnostic for DESIGN.md §11."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import pynvml  # noqa: E402
import torch  # noqa: E402

pynvml.nvmlInit()
vis = os.environ.get("CUDA_VISIBLE_DEVICES")
h = pynvml.nvmlDeviceGetHandleByIndex(int(vis.split(",")[0]) if vis else 0)
E = lambda: pynvml.nvmlDeviceGetTotalEnergyConsumption(h)  # noqa: E731
torch.cuda.init()
time.sleep(1.0)
e0, t0 = E(), time.perf_counter()
time.sleep(2.0)
print(f"idle: {(E() - e0) / (time.perf_counter() - t0) / 1e3:.1f} W")
for n_el in (1 << 29, 1 << 30):
    a = torch.randn(n_el, device="cuda").to(torch.bfloat16)
    b = torch.empty_like(a)
    for _ in range(20):
        b.copy_(a)
    torch.cuda.synchronize()
    st, en = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0 = E()
    st.record()
    n, t_end = 0, time.perf_counter() + 1.5
    while time.perf_counter() < t_end:
        b.copy_(a)
        n += 1
    en.record()
    torch.cuda.synchronize()
    mj = E() - e0
    ms = st.elapsed_time(en)
    gb = n * 2 * a.numel() * 2 / 1e9
    print(f"copy {a.numel() * 2 / 2**30:.0f} GiB: {gb / (ms / 1e3):.0f} GB/s, {mj / ms:.0f} W, {mj / gb:.1f} mJ/GB "
          f"({mj * 1e9 / (gb * 1e9 * 8) :.1f} pJ/bit board)", flush=True)
    del a, b
    torch.cuda.empty_cache()
