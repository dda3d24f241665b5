"""Cost of one block-cyclic round's pieces at several chunk sizes (developer tool)."""
import sys, os, ctypes, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
k, s = 4, 4
x = synth.make_torch(1 << 27, "i64", "uniform", device="cuda"); y = torch.empty_like(x)
pb = S.sam_shard_payload_bytes(1, k, s)
pay = torch.zeros(pb, dtype=torch.uint8, device="cuda")
seed = torch.zeros(k * s, dtype=torch.int64, device="cuda")
P = lambda t: ctypes.c_void_p(t.data_ptr())
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
def t(fn, it=20):
    fn(); torch.cuda.synchronize(); e0.record()
    for _ in range(it): fn()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it * 1000
for lc in (20, 22, 24, 26):
    c = 1 << lc
    ts = t(lambda: S.sam_shard_state(1, k, s, P(x), c, 0, P(pay)))
    tq = t(lambda: S.sam_scan_seeded(1, k, s, 1, P(x), P(y), c, 0, P(seed), None))
    tp = t(lambda: S.sam_scan(1, k, s, 1, P(x), P(y), c))
    tf = t(lambda: S.sam_cyclic_fold(1, k, s, P(pay), 0, 1, P(seed), P(seed), P(seed)))
    def rnd():
        S.sam_shard_state(1, k, s, P(x), c, 0, P(pay)); S.sam_cyclic_fold(1, k, s, P(pay), 0, 1, P(seed), P(seed), P(seed))
        S.sam_scan_seeded(1, k, s, 1, P(x), P(y), c, 0, P(seed), None)
    tr = t(rnd)
    t0 = time.perf_counter(); [S.sam_cyclic_fold(1, k, s, P(pay), 0, 1, P(seed), P(seed), P(seed)) for _ in range(1000)]; th = (time.perf_counter() - t0) * 1e3
    torch.cuda.synchronize()
    print(f"chunk 2^{lc} ({c*8/2**20:.0f} MiB): state {ts:.1f} us  seeded scan {tq:.1f} us  plain scan {tp:.1f} us  fold {tf:.1f} us  round {tr:.1f} us  "
          f"(ideal 2w/BW {2*c*8/6.5e6:.1f} us)  host per fold call {th:.1f} us", flush=True)
