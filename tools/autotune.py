"""Install-time autotuner (SAM's: "runs when SAM is installed and determines the optimal
number of input elements to allocate to each thread for different ranges of problem sizes").
For each (element type, order, tuple) class and problem-size range it times the carry unit
(tiles per super-tile M) x pipeline depth x fold variant through sam_tune_override and writes the
fastest to paper_conf_pldi_malekiyb16_b200/lib/sam_tune.txt, which libsam.so reads at first use.
    python tools/autotune.py [--quick]"""
import os, statistics, sys, itertools
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402

quick = "--quick" in sys.argv
OUT = next((a.split("=", 1)[1] for a in sys.argv if a.startswith("--out=")),
           os.path.join(os.path.dirname(S.LIB_PATH), "sam_tune.txt"))
TY = {"i32": "u32", "i64": "u64", "f32": "f32", "f64": "f64"}
classes = [(dt, k, s) for dt in ("i32", "i64") for k in (1, 2, 3, 4, 5, 6, 7, 8) for s in (1, 2, 3, 4, 5, 6, 7, 8)
           if k * s <= 16 or (k, s) in ((4, 4), (2, 8), (8, 2), (8, 8))]
classes += [(dt, 1, s) for dt in ("f32", "f64") for s in (1, 2, 4, 8)]
if quick:
    classes = [c for c in classes if c[1] in (1, 2, 4, 8) and c[2] in (1, 2, 4, 8)]
ranges = [(20, 24, 22), (25, 28, 28), (29, 33, 30)]  # (log2 lo, log2 hi, measured at)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
lines = []
bufs = {}
for lo, hi, lg in ranges:
    for dt, k, s in classes:
        n = 1 << lg
        key = (dt, lg)
        if key not in bufs:
            bufs.clear()
            torch.cuda.empty_cache()
            x = synth.make_torch(n, dt, "uniform" if dt[0] == "i" else "unif01", device="cuda")
            bufs[key] = (x, torch.empty_like(x))
        x, y = bufs[key]
        best = None
        for M, lag, vf in itertools.product((0, 1, 2, 3, 4), (0, 6, 8, 12), (-1,) if k == 1 else (0, 1)):
            S.sam_tune_override(M if M else -1, lag if lag else -1, vf, -1, -1)
            try:
                for _ in range(2):
                    S.scan(x, k, s, True, out=y)
                torch.cuda.synchronize()
                ts = []
                for _ in range(3):
                    e0.record()
                    for _ in range(3):
                        S.scan(x, k, s, True, out=y)
                    e1.record()
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1) / 3)
            except Exception as ex:  # a combination the kernel rejects
                continue
            t = statistics.median(ts)
            if best is None or t < best[0]:
                best = (t, M, lag, vf)
        S.sam_tune_override(-1, -1, -1, -1, -1)
        t, M, lag, vf = best
        vfield = 0 if vf < 0 else vf + 1
        lines.append(f"{TY[dt]} {k} {s} {lo} {hi} {M} {lag} {vfield} 0")
        print(f"{dt} k={k} s={s} 2^{lg}: {2 * n * x.element_size() / (t * 1e-3) / 1e9:.0f} GB/s  M={M} lag={lag} vfold={vf}",
              flush=True)
with open(OUT, "w") as f:
    f.write("# sam_tune.txt -- written by tools/autotune.py on " + torch.cuda.get_device_name() + "\n")
    f.write("# type k s log2n_lo log2n_hi M lag vfold land   (0 = default; vfold/land 1 = off, 2 = on)\n")
    f.write("\n".join(lines) + "\n")
print("wrote", OUT)
