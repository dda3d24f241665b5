"""Per-tile pipeline event trace (developer tool): python tools/trace_tiles.py i32 28 1 1"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
dt, logn, k, s = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
n = 1 << logn
x = synth.make_torch(n, dt, "uniform", device="cuda"); y = torch.empty_like(x)
import time
soak = float(os.environ.get("SOAK_S", "0"))  # sustained-load clocks (power cap) before the traced launch
t0 = time.time()
while True:
    for _ in range(3): S.scan(x, k, s, True, out=y)
    torch.cuda.synchronize()
    if time.time() - t0 >= soak: break
tr = torch.zeros(16 * (n // 1000 + 16), dtype=torch.int64, device="cuda")
S.lib().sam_debug_set_trace(ctypes.c_void_p(tr.data_ptr()))
S.scan(x, k, s, True, out=y); torch.cuda.synchronize()
S.lib().sam_debug_set_trace(None)
t = tr.cpu().numpy().reshape(-1, 16)
t = t[t[:, 0] > 0]
t0 = t[:, 0].min()
ts_cols = [0, 1, 2, 3, 4, 5, 6, 7, 8, 9, 10, 13, 14]  # timestamp events (11, 12: counters)
tf = np.full(t.shape, np.nan)
for c in range(16):
    nz = t[:, c] != 0
    tf[nz, c] = (t[nz, c] - t0).astype(np.float64) if c in ts_cols else t[nz, c]
extra = tf[:, 8:].copy()
extra[np.isnan(extra)] = 0
t = tf[:, :8]  # ns since the first claim; NaN = event not recorded for this tile
names = ["claim", "p1start", "p1done", "aggpub", "lbstart", "inclpub", "p2start", "stored"]
print(f"{dt} 2^{logn} k={k} s={s}: tiles {len(t)}  span {np.nanmax(t)/1e3:.1f} us  rate {len(t)/(np.nanmax(t)/1e3):.1f} tiles/us")
def q(a):
    a = np.asarray(a, dtype=np.float64); a = a[~np.isnan(a)]
    return " ".join(f"{np.percentile(a, pp):7.2f}" for pp in (10, 50, 90, 99)) if a.size else "n/a"
print("interval (us)            p10     p50     p90     p99")
for a_, b_ in [(0, 1), (1, 2), (2, 3), (3, 4), (4, 5), (5, 6), (6, 7), (0, 3), (3, 5), (0, 7)]:
    d = (t[:, b_] - t[:, a_]) / 1e3
    print(f"{names[a_]:>8} -> {names[b_]:<8} {q(d)}")
d = (t[:-1, 3] - t[1:, 3]) / 1e3
print(f"agg(t-1) - agg(t)        {q(d)}")
d = (t[:-1, 5] - t[1:, 3]) / 1e3
print(f"incl(t-1) - agg(t)       {q(d)}")
# parked footprint: tiles between claim (HBM load issued) and carry application start (L2 reload done)
tile_bytes = x.element_size() * (n // max(1, len(t)))
ev = np.concatenate([np.stack([t[:, 0], np.ones(len(t))], 1), np.stack([t[:, 6], -np.ones(len(t))], 1)])
ev = ev[np.argsort(ev[:, 0], kind="stable")]
occ = np.cumsum(ev[:, 1])
print(f"parked tiles: p50 {np.percentile(occ, 50):.0f}  p90 {np.percentile(occ, 90):.0f}  max {occ.max():.0f}"
      f"  (~{np.percentile(occ, 50) * tile_bytes / 2**20:.1f} / {occ.max() * tile_bytes / 2**20:.1f} MiB)")
lb = extra[extra[:, 0] != 0]
if len(lb):
    print(f"look-back units {len(lb)}: first poll RTT {q((lb[:,1]-lb[:,0])/1e3)}  loop {q((lb[:,2]-lb[:,0])/1e3)}  polls {q(lb[:,3])}  stop=own-prev {lb[:,4].mean():.2f}")
# super-tile view: aggregate of its last sub-tile -> carry team starts -> first sub-tile's carry ready
first = np.nonzero(~np.isnan(t[:, 4]))[0]
if len(first) > 2:
    M = int(np.median(np.diff(first)))
    f = first[first + M - 1 < len(t)]
    last = f + M - 1
    us = lambda a: np.asarray(a) / 1e3
    print(f"super-tiles (M={M}):  lastagg->lbstart {q(us(t[f, 4] - t[last, 3]))}   lbstart->incl {q(us(t[f, 5] - t[f, 4]))}")
    e = tf[f]
    print(f"  lbstart->poll0 {q(us(e[:, 8] - e[:, 4]))}  poll0->lbdone {q(us(e[:, 10] - e[:, 8]))}  lbdone->barrier {q(us(e[:, 13] - e[:, 10]))}"
          f"  barrier->handoff {q(us(e[:, 14] - e[:, 13]))}  handoff->incl0 {q(us(e[:, 5] - e[:, 14]))}")
# skew: when did the last aggregate a super-tile's fold needs (super-tiles S-P+1..S-1) appear, relative to
# the super-tile's own last aggregate and to its fold start / end
if len(first) > 2:
    P = int(os.environ.get("P", "148"))
    lastagg = t[last, 3]
    ns = len(f)
    need = np.full(ns, np.nan)
    for i in range(ns):
        lo = max(0, i - P + 1)
        if i > lo: need[i] = np.nanmax(lastagg[lo:i])
    e = tf[f]
    print(f"skew: need-ownagg {q(us(need - lastagg))}  need-poll0 {q(us(need - e[:, 8]))}  lbdone-need {q(us(e[:, 10] - need))}")
    # per-CTA progress spread: for each round, max - min of the super-tiles' own last aggregate
    R = ns // P
    if R > 2:
        la = lastagg[:R * P].reshape(R, P)
        print(f"round spread of own-agg (max-min over CTAs) {q(us(np.nanmax(la, 1) - np.nanmin(la, 1)))}")
        d = np.diff(np.nanmedian(la, 1))
        print(f"round period (median own-agg) {q(us(d))}")
