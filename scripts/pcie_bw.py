"""Pinned host<->device copy bandwidth on the box (context for the e2e path)."""
import torch, time
for mb in (2, 64, 256):
    n = mb * 2**20 // 8
    h = torch.empty(n, dtype=torch.float64).pin_memory()
    d = torch.empty(n, dtype=torch.float64, device="cuda")
    for name, f in (("H2D", lambda: d.copy_(h, non_blocking=True)), ("D2H", lambda: h.copy_(d, non_blocking=True))):
        f(); torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(10): f()
        b.record(); torch.cuda.synchronize()
        print(f"{name} {mb} MB: {10 * mb / 1024 / (a.elapsed_time(b) / 1000):.1f} GiB/s")
