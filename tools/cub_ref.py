"""Context: torch.cumsum (CUB DeviceScan underneath) throughput on this GPU (developer tool)."""
import torch
for dt, logn in ((torch.int32, 30), (torch.int32, 28), (torch.int64, 28), (torch.float32, 28)):
    n = 1 << logn
    x = torch.randint(-100, 100, (n,), dtype=dt, device="cuda") if not dt.is_floating_point else torch.rand(n, device="cuda")
    y = torch.empty_like(x)
    for _ in range(3): torch.cumsum(x, 0, dtype=dt, out=y)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20): torch.cumsum(x, 0, dtype=dt, out=y)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 20
    print(f"torch.cumsum {dt} 2^{logn}: {ms:.3f} ms {n/ms/1e6:.1f} Gval/s {2*n*x.element_size()/ms/1e6:.0f} GB/s", flush=True)
