"""Repeat-median throughput sweep over the benchmark configs (developer tool).
    python tools/sweep.py [reps]"""
import sys, os, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import time
import torch, synth
SOAK = float(os.environ.get("SOAK", "0"))
import paper_conf_pldi_malekiyb16_b200 as S
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
cfgs = [("i32", 30, 1, 1), ("i32", 28, 1, 1), ("i64", 28, 1, 1), ("i32", 28, 2, 1), ("i64", 28, 2, 1),
        ("i32", 28, 4, 1), ("i64", 28, 4, 1), ("i32", 28, 8, 1), ("i64", 28, 8, 1), ("i64", 28, 1, 2),
        ("i64", 28, 1, 3), ("i64", 28, 1, 5), ("i64", 28, 1, 8), ("i64", 28, 2, 8), ("i64", 28, 4, 4),
        ("f32", 28, 1, 4), ("f64", 28, 1, 1)]
if len(sys.argv) > 2:  # optional filter: "i32:30:1:1,i64:28:1:8"
    want = [tuple(int(v) if i else v for i, v in enumerate(c.split(":"))) for c in sys.argv[2].split(",")]
    cfgs = want  # in the order given
data = {}
for c in cfgs:
    dt, logn, k, s = c
    x = synth.make_torch(1 << logn, dt, "uniform", device="cuda"); y = torch.empty_like(x)
    data[c] = (x, y)
res = {c: [] for c in cfgs}
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for r in range(reps):
    for c in cfgs:
        dt, logn, k, s = c
        x, y = data[c]
        for _ in range(2): S.scan(x, k, s, True, out=y)
        if SOAK > 0:  # sustained: run the config alone for SOAK seconds first (power-cap clocks)
            t0 = time.time()
            while time.time() - t0 < SOAK:
                for _ in range(5): S.scan(x, k, s, True, out=y)
                torch.cuda.synchronize()
        torch.cuda.synchronize(); e0.record()
        it = 10
        for _ in range(it): S.scan(x, k, s, True, out=y)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / it
        res[c].append(2 * (1 << logn) * x.element_size() / ms / 1e6)
for c in cfgs:
    v = res[c]
    print(f"{c[0]} 2^{c[1]} k={c[2]} s={c[3]}: median {statistics.median(v):6.0f} GB/s  ({min(v):.0f}-{max(v):.0f})", flush=True)
