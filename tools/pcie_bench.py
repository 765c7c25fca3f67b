"""Pinned host<->device copy bandwidth (dev tool): H2D, D2H, and both concurrently."""
import time

import torch

n = 4 << 30
h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
d1 = torch.empty(n, dtype=torch.uint8, device="cuda")
d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for name, fn in [("h2d", lambda: d1.copy_(h1, non_blocking=True)),
                 ("d2h", lambda: h2.copy_(d2, non_blocking=True))]:
    fn(); torch.cuda.synchronize()
    t = time.perf_counter(); fn(); torch.cuda.synchronize(); dt = time.perf_counter() - t
    print(f"{name}: {n / dt / 1e9:.1f} GB/s")
torch.cuda.synchronize()
t = time.perf_counter()
with torch.cuda.stream(s1):
    d1.copy_(h1, non_blocking=True)
with torch.cuda.stream(s2):
    h2.copy_(d2, non_blocking=True)
torch.cuda.synchronize()
dt = time.perf_counter() - t
print(f"bidirectional: {2 * n / dt / 1e9:.1f} GB/s total ({n / dt / 1e9:.1f} each way)")
