"""Carry-scheme ablation on B200 (the paper's Sec. 5.4): the same
generic kernel under SAM's static schedule, decoupled look-back and the chained scheme, next to the
production kernel (warp-specialised, SAM static schedule), on C2 / C3 / C4-shaped inputs.
    python tools/ablation.py [out.json]
Kernel time by CUDA events (median of 5 after 2 warm-ups), inputs resident in HBM."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402

CFGS = [("C2 i32 k=1 s=1", "i32", 30, 1, 1), ("C3 i32 k=2 s=1", "i32", 28, 2, 1), ("C3 i32 k=8 s=1", "i32", 28, 8, 1),
        ("C3 i64 k=4 s=1", "i64", 28, 4, 1), ("C4 i64 k=1 s=4", "i64", 28, 1, 4), ("C4 i64 k=1 s=8", "i64", 28, 1, 8)]
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)


def timeit(fn, reps=5):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


out = []
for name, dt, logn, k, s in CFGS:
    n = 1 << logn
    x = synth.make_torch(n, dt, "uniform", device="cuda")
    y = torch.empty_like(x)
    w = x.element_size()
    row = {"config": name, "n": n}
    row["production_static"] = timeit(lambda: S.scan(x, k, s, True, out=y))
    for carry in ("static", "lookback", "chained"):
        nn = n if carry != "chained" else min(n, 1 << 24)  # the serial chain: bounded size
        xv, yv = x[:nn], y[:nn]
        ms = timeit(lambda: S.scan_op(xv, "add", k, s, True, out=yv, carry=carry), reps=3 if carry == "chained" else 5)
        row[f"generic_{carry}"] = ms * n / nn  # scaled to the full n for comparison
        if carry == "chained":
            row["chained_n"] = nn
    for key in ("production_static", "generic_static", "generic_lookback", "generic_chained"):
        row[key + "_gbs"] = 2 * w * n / (row[key] * 1e-3) / 1e9
    out.append(row)
    print(json.dumps(row), flush=True)
    del x, y
    torch.cuda.empty_cache()
if len(sys.argv) > 1:
    json.dump(out, open(sys.argv[1], "w"), indent=1)
