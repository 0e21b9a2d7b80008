"""Pinned host <-> device copy bandwidth on this box (context for e2e)."""
import torch
n = 8 << 20
h = torch.empty(n, dtype=torch.uint8).pin_memory()
h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
h.fill_(1)
h2.fill_(2)
for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)),
                 ("d2h", lambda: h.copy_(d, non_blocking=True)),
                 ("h2d again", lambda: d.copy_(h, non_blocking=True))):
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(50):
        fn()
    e1.record()
    torch.cuda.synchronize()
    print(f"{name}: {50 * n / (e0.elapsed_time(e1) * 1e-3) / 1e9:.1f} GB/s")
torch.cuda.synchronize()
import time
t0 = time.perf_counter()
for _ in range(50):
    with torch.cuda.stream(s1):
        d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2):
        h2.copy_(d2, non_blocking=True)
torch.cuda.synchronize()
dt = time.perf_counter() - t0
print(f"concurrent h2d+d2h: {50 * n / dt / 1e9:.1f} GB/s each direction")
