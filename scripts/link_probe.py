"""Host link bandwidth on the GPU box: pinned H2D, D2H, and both at once on two streams (1 GiB each)."""
import torch
N = 1 << 28  # int32 elements = 1 GiB
h1 = torch.empty(N, dtype=torch.int32).pin_memory(); h2 = torch.empty(N, dtype=torch.int32).pin_memory()
d1 = torch.empty(N, dtype=torch.int32, device="cuda"); d2 = torch.empty(N, dtype=torch.int32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(f, reps=5):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize(); e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); f(); torch.cuda.synchronize(); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best
gb = 4 * N / 1e9
ms = t(lambda: d1.copy_(h1, non_blocking=True)); print(f"H2D {gb / ms * 1e3:.1f} GB/s")
ms = t(lambda: h1.copy_(d1, non_blocking=True)); print(f"D2H {gb / ms * 1e3:.1f} GB/s")
def both():
    with torch.cuda.stream(s1): d1.copy_(h1, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
ms = t(both); print(f"H2D + D2H concurrently: {2 * gb / ms * 1e3:.1f} GB/s total ({gb / ms * 1e3:.1f} each way)")
