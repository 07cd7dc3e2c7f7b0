"""Microbenchmark: L2-resident vs HBM copy bandwidth on this GPU (torch copy_, CUDA events)."""
import torch
for mib in (8, 16, 32, 48, 64, 96, 256, 2048):
    n = (mib << 20) // 2
    a = torch.randn(n, device="cuda", dtype=torch.float32).to(torch.bfloat16)
    b = torch.empty_like(a)
    for _ in range(5):
        b.copy_(a)
    reps = max(5, int(20000 / mib))
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s.record()
    for _ in range(reps):
        b.copy_(a)
    e.record()
    torch.cuda.synchronize()
    t = s.elapsed_time(e) / reps * 1e-3
    print("copy %5d MiB: %.0f GB/s (read+write)" % (mib, 2 * (mib << 20) / t / 1e9), flush=True)
