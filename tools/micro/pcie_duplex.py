"""Host link ceiling for the e2e path: pinned H2D alone, D2H alone, and both at once on two
streams (1.6 GB each way, the per-step volume of H).  Not part of the library."""
import time

import torch

n = 1610612736 // 4
h_src = torch.empty(n, dtype=torch.float32).pin_memory()
h_dst = torch.empty(n, dtype=torch.float32).pin_memory()
d_a = torch.empty(n, dtype=torch.float32, device="cuda")
d_b = torch.empty(n, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def run(h2d, d2h, reps=5):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        if h2d:
            with torch.cuda.stream(s1):
                d_a.copy_(h_src, non_blocking=True)
        if d2h:
            with torch.cuda.stream(s2):
                h_dst.copy_(d_b, non_blocking=True)
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


run(True, True, 2)
for name, a, b in (("h2d", True, False), ("d2h", False, True), ("both", True, True)):
    t = run(a, b)
    gb = (a + b) * n * 4 / 1e9
    print(f"{name}: {t * 1e3:.1f} ms per 1.61 GB each way, {gb / t:.1f} GB/s total")
