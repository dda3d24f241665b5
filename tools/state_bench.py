"""State pass (sam_shard_state) vs the scan on the same input (developer tool):
    python tools/state_bench.py        (SAM_STATE_VIA_SCAN=1: the scan kernel in state-only mode)"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
def t(fn, it=10):
    fn(); torch.cuda.synchronize(); e0.record()
    for _ in range(it): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it * 1000
P = lambda t_: ctypes.c_void_p(t_.data_ptr())
for dt, logn, k, s in [("i32", 28, 1, 1), ("i64", 28, 1, 1), ("i32", 28, 8, 1), ("i64", 28, 4, 4), ("i64", 28, 8, 1),
                       ("i64", 28, 2, 8), ("f32", 28, 1, 4), ("i64", 30, 4, 4), ("i64", 22, 4, 4), ("i32", 22, 1, 1)]:
    n = 1 << logn
    x = synth.make_torch(n, dt, "uniform", device="cuda"); y = torch.empty_like(x)
    dc = S.dtype_code(x.dtype)
    pay = torch.zeros(S.sam_shard_payload_bytes(dc, k, s), dtype=torch.uint8, device="cuda")
    ts = t(lambda: S.sam_shard_state(dc, k, s, P(x), n, 0, P(pay)))
    tq = t(lambda: S.sam_scan(dc, k, s, 1, P(x), P(y), n))
    w = x.element_size()
    print(f"{dt} 2^{logn} k={k} s={s}: state {ts:8.1f} us ({n*w/ts/1e3:6.0f} GB/s read)  scan {tq:8.1f} us  state/scan {ts/tq:.2f}", flush=True)
    del x, y
