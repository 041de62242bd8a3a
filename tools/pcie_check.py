"""Pinned host <-> device copy rates on this box (context for the bench's e2e number)."""
import time
import torch
n = 2 * 1024**3
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for _ in range(2):
    d.copy_(h, non_blocking=True); torch.cuda.synchronize()
t0 = time.perf_counter(); d.copy_(h, non_blocking=True); torch.cuda.synchronize(); t1 = time.perf_counter()
h.copy_(d, non_blocking=True); torch.cuda.synchronize(); t2 = time.perf_counter()
print(f"H2D {n / (t1 - t0) / 1e9:.1f} GB/s, D2H {n / (t2 - t1) / 1e9:.1f} GB/s")
