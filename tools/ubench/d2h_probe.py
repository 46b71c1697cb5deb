"""Where does the e2e host-depth time go on C2 (n = 2^24)?  D2H of n bytes from
device to pinned host (1 or 8 chunks), n/2 bytes (4-bit codes), and the host
int8 -> int32 widening (numpy, one thread) into a pinned int32 array."""
import os, time
import numpy as np
import torch

n = 1 << 24
dev8 = torch.zeros(n, dtype=torch.int8, device="cuda")
h8 = torch.empty(n, dtype=torch.int8, pin_memory=True)
h32 = torch.empty(n, dtype=torch.int32, pin_memory=True)
s = torch.cuda.Stream()
def t_copy(nbytes, chunks):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s)
        for c in range(chunks):
            a, b = nbytes * c // chunks, nbytes * (c + 1) // chunks
            h8[a:b].copy_(dev8[a:b], non_blocking=True)
        e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)
for _ in range(3): t_copy(n, 1)
for nb, ch in ((n, 1), (n, 8), (n // 2, 1), (n // 2, 8), (4 * n // 1, 1) if False else (n, 16)):
    ms = min(t_copy(nb, ch) for _ in range(5))
    print(f"D2H {nb/1e6:.1f} MB in {ch} chunks: {ms:.3f} ms = {nb/ms/1e6:.1f} GB/s")
a8 = h8.numpy(); a32 = h32.numpy()
for _ in range(2): np.copyto(a32, a8)
t0 = time.perf_counter(); np.copyto(a32, a8); t1 = time.perf_counter()
print(f"host widen int8->int32 1 thread: {(t1-t0)*1e3:.3f} ms; cpus {os.cpu_count()}")
