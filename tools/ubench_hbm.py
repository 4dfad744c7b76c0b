"""HBM ceilings on this B200 for the access mixes of the two GEMM kernels (torch ops, CUDA events):
write-only (fill), read-only (sum), copy (1:1), and read+write at GEMM1's 1:4 and GEMM2's 10:1 ratios."""
import torch

torch.cuda.init()
N = 1 << 29  # 512 MiB


def t(fn, reps=20):
    for _ in range(3):
        fn()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    ts = []
    for _ in range(reps):
        a.record(); fn(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2] * 1e-3


x = torch.empty(N, dtype=torch.uint8, device="cuda")
y = torch.empty(N, dtype=torch.uint8, device="cuda")
s = t(lambda: x.fill_(1)); print(f"write-only fill 512 MiB: {N / s / 1e9:.0f} GB/s")
xf = x.view(torch.float32)
s = t(lambda: xf.sum()); print(f"read-only sum 512 MiB:   {N / s / 1e9:.0f} GB/s")
s = t(lambda: y.copy_(x)); print(f"copy 512 MiB:            {2 * N / s / 1e9:.0f} GB/s")
# 1:4 read:write (GEMM1: Q,K in, X' out): read a 128 MiB slice, write 4 slices
src = x[: N // 4]
dst = y.view(4, N // 4)
s = t(lambda: dst.copy_(src.unsqueeze(0).expand(4, -1))); print(f"1:4 read:write:          {(N // 4 + N) / s / 1e9:.0f} GB/s")
