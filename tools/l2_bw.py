"""Measure L2-resident copy bandwidth vs HBM copy bandwidth (developer tool)."""
import torch
for mb in (8, 16, 32, 48, 64, 4096):
    n = mb * (1 << 20) // 4
    x = torch.ones(n, device="cuda"); y = torch.empty_like(x)
    for _ in range(5): y.copy_(x)
    torch.cuda.synchronize()
    reps = 200 if mb < 1000 else 10
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps): y.copy_(x)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    print(f"copy {mb} MB: {ms*1e3:.1f} us  {2*n*4/ms/1e6:.0f} GB/s", flush=True)
    # read-only: sum
    for _ in range(3): x.sum()
    torch.cuda.synchronize(); e0.record()
    for _ in range(reps): x.sum()
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    print(f"  read {mb} MB: {ms*1e3:.1f} us  {n*4/ms/1e6:.0f} GB/s", flush=True)
