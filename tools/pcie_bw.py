"""Host<->device copy bandwidth from pinned memory (the bound of bench.py's e2e copies)."""
import time
import torch

n = 120 * 1024 * 1024 // 8
h = torch.empty(n, dtype=torch.float64).pin_memory()
d = torch.empty(n, dtype=torch.float64, device="cuda")
for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)),
                 ("d2h", lambda: h.copy_(d, non_blocking=True))):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(10):
        fn()
    torch.cuda.synchronize()
    el = (time.perf_counter() - t0) / 10
    print(f"{name}: {n * 8 / el / 1e9:.1f} GB/s ({n * 8 / 1e6:.0f} MB in {el * 1e3:.2f} ms)")
