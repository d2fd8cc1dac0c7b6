"""Pinned host <-> device copy bandwidth (1 GiB), one direction and both concurrently."""
import torch, time
n = 1 << 28  # floats = 1 GiB
h = torch.empty(n, dtype=torch.float32).pin_memory()
h2 = torch.empty(n, dtype=torch.float32).pin_memory()
d = torch.empty(n, dtype=torch.float32, device="cuda")
d2 = torch.empty(n, dtype=torch.float32, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def timeit(fn, reps=5):
    fn(); torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(reps): fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t) / reps
gb = 4 * n / 1e9
t = timeit(lambda: d.copy_(h, non_blocking=True)); print(f"H2D {gb / t:.1f} GB/s")
t = timeit(lambda: h.copy_(d, non_blocking=True)); print(f"D2H {gb / t:.1f} GB/s")
def both():
    with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
t = timeit(both); print(f"concurrent: {gb / t:.1f} GB/s each direction")
