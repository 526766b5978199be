"""Pinned host -> device bandwidth with 1 / 2 / 4 concurrent copy streams (the
end-to-end path is PCIe-bound)."""
import time
import torch
N = 64 << 20
for k in (1, 2, 4):
    xs = [torch.empty(N // k, dtype=torch.uint8).pin_memory() for _ in range(k)]
    ds = [torch.empty(N // k, dtype=torch.uint8, device="cuda") for _ in range(k)]
    ss = [torch.cuda.Stream() for _ in range(k)]
    for _ in range(3):
        for x, d, s in zip(xs, ds, ss):
            with torch.cuda.stream(s):
                d.copy_(x, non_blocking=True)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(10):
        for x, d, s in zip(xs, ds, ss):
            with torch.cuda.stream(s):
                d.copy_(x, non_blocking=True)
    torch.cuda.synchronize()
    print("%d stream(s): %.1f GB/s" % (k, 10 * N / (time.perf_counter() - t0) / 1e9))
