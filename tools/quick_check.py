"""Quick GPU sanity + timing check (developer tool)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_pldi_malekiyb16_b200 as S

def check(dt, n, k, s, incl):
    xn = synth.make(n, dt, "uniform" if dt in ("i32", "i64") else "unif01", seed=n + k * 8 + s)
    x = torch.from_numpy(xn).cuda()
    y = S.scan(x, k, s, incl); torch.cuda.synchronize()
    ref = oracle.scan(xn, k, s, incl)[0]
    got = y.cpu().numpy().view(ref.dtype) if dt in ("i32","i64") else y.cpu().numpy()
    ok = np.array_equal(got, ref) if dt in ("i32","i64") else np.allclose(got, ref, rtol=1e-4)
    print(f"{dt} n={n} k={k} s={s} incl={incl}: {'OK' if ok else 'FAIL'}", flush=True)
    if not ok and dt in ("i32","i64"):
        bad = np.nonzero(got != ref)[0]; print("  first bad", bad[:10], got[bad[:3]], ref[bad[:3]])
    return ok

for args in [("i32", 1000, 1, 1, True), ("i32", 100000, 1, 1, True), ("i32", 100000, 2, 1, True),
             ("i32", 100000, 1, 2, True), ("i32", 100000, 1, 3, True), ("i64", 100000, 4, 4, True),
             ("i32", 100000, 3, 1, False), ("i64", 1<<21, 8, 8, True), ("f32", 100000, 1, 1, True)]:
    check(*args)

def bench(dt, n, k, s, iters=20):
    x = synth.make_torch(n, dt, "uniform", device="cuda")
    y = torch.empty_like(x)
    for _ in range(3): S.scan(x, k, s, True, out=y)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters): S.scan(x, k, s, True, out=y)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / iters
    gbs = 2 * n * x.element_size() / ms / 1e6
    print(f"bench {dt} n={n} k={k} s={s}: {ms:.3f} ms  {n/ms/1e6:.1f} Gval/s  {gbs:.0f} GB/s", flush=True)

def memcpy(n, w, iters=20):
    a = torch.empty(n * w, dtype=torch.uint8, device="cuda"); b = torch.empty_like(a)
    for _ in range(3): b.copy_(a)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters): b.copy_(a)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / iters
    print(f"memcpy {n*w/2**30:.1f} GiB: {ms:.3f} ms {2*n*w/ms/1e6:.0f} GB/s", flush=True)

if "--bench" in sys.argv:
    memcpy(1 << 30, 4)
    bench("i32", 1 << 30, 1, 1)
    for k in (1, 2, 4, 8):
        bench("i32", 1 << 28, k, 1)
        bench("i64", 1 << 28, k, 1)
    for s in (2, 3, 4, 5, 8):
        bench("i64", 1 << 28, 1, s)
    bench("i64", 1 << 28, 4, 4)
