"""Host<->device copy bandwidth, one direction at a time and both together
(full duplex?), pinned memory, 1 GiB per copy; tuning helper for the e2e path."""
import time
import torch

n = 1 << 30
h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
d1 = torch.empty(n, dtype=torch.uint8, device="cuda")
d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn):
    torch.cuda.synchronize()
    t = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    return time.perf_counter() - t


for _ in range(2):
    th = timed(lambda: d1.copy_(h1, non_blocking=True))
    td = timed(lambda: h2.copy_(d2, non_blocking=True))

    def both():
        with torch.cuda.stream(s1):
            d1.copy_(h1, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
    tb = timed(both)
print(f"H2D {n / th / 1e9:.1f} GB/s  D2H {n / td / 1e9:.1f} GB/s  both together {2 * n / tb / 1e9:.1f} GB/s total")
