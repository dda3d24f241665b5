"""Small-n (launch-bound) timings of the production kernel vs the generic kernel's carry schemes (developer tool)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
def t(fn, it=50):
    for _ in range(5): fn()
    torch.cuda.synchronize(); e0.record()
    for _ in range(it): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it * 1000
for dt, logn, k, s in [("i32", 16, 1, 1), ("i32", 18, 1, 1), ("i32", 20, 1, 1), ("i32", 22, 1, 1), ("i32", 20, 4, 1), ("i64", 20, 4, 4)]:
    n = 1 << logn
    x = synth.make_torch(n, dt, "uniform", device="cuda"); y = torch.empty_like(x)
    tp = t(lambda: S.scan(x, k, s, True, out=y))
    tl = t(lambda: S.scan_op(x, "add", k, s, True, out=y, carry="lookback"))
    ts = t(lambda: S.scan_op(x, "add", k, s, True, out=y, carry="static"))
    tm = t(lambda: y.copy_(x))
    print(f"{dt} 2^{logn} k={k} s={s}: production {tp:6.1f} us  generic look-back {tl:6.1f} us  generic static {ts:6.1f} us  copy {tm:5.1f} us", flush=True)
