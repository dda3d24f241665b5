"""Per-GPU cost of the block-cyclic schedule (NEXT-1) vs the single-pass scan and vs contiguous
shards, on one GPU (developer tool): python tools/cyclic_bench.py [logn] [k] [s]"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
from paper_conf_pldi_malekiyb16_b200.dist import scan_cyclic_virtual, scan_virtual_shards
logn = int(sys.argv[1]) if len(sys.argv) > 1 else 30
k = int(sys.argv[2]) if len(sys.argv) > 2 else 4
s = int(sys.argv[3]) if len(sys.argv) > 3 else 4
n = 1 << logn
x = synth.make_torch(n, "i64", "uniform", device="cuda"); y = torch.empty_like(x)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
def t(fn, it=3):
    fn(); torch.cuda.synchronize(); e0.record()
    for _ in range(it): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it
ms = t(lambda: S.scan(x, k, s, True, out=y))
print(f"single-pass scan: {ms:.2f} ms  {n/ms/1e6:.0f} Gvalues/s", flush=True)
for p in (8,):
    b = [i * n // p for i in range(p + 1)]
    ms = t(lambda: scan_virtual_shards(x, b, k, s, True))
    print(f"contiguous shards p={p} (all on one GPU): {ms:.2f} ms  per-GPU-equivalent {n/ms/1e6:.0f} Gvalues/s", flush=True)
for logc in (20, 21, 22, 23, 24):
    for la in (0, 1):
        ms = t(lambda: scan_cyclic_virtual(x, 1, 1 << logc, k, s, True, lookahead=la))
        print(f"cyclic p=1 chunk 2^{logc} lookahead {la}: {ms:.2f} ms  {n/ms/1e6:.0f} Gvalues/s", flush=True)
for logc in (21, 22):
    ms = t(lambda: scan_cyclic_virtual(x, 8, 1 << logc, k, s, True, lookahead=1))
    print(f"cyclic p=8 virtual chunk 2^{logc}: {ms:.2f} ms  {n/ms/1e6:.0f} Gvalues/s (all ranks' work on one GPU)", flush=True)
