"""Find failing/hanging configs quickly (developer tool). Each config runs in a subprocess with a timeout."""
import subprocess, sys, os
cfgs = sys.argv[1:] or ["i32:20011:1:1", "i64:20011:1:1", "i32:20011:8:1", "i64:20011:8:8", "i64:20011:4:4",
                        "f32:20011:3:3", "i32:2109497:1:1", "i64:2109497:8:8", "i32:268435456:1:1", "i32:1073741824:1:1"]
code = r'''
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch, synth, oracle
import paper_conf_pldi_malekiyb16_b200 as S
dt, n, k, s = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
x = synth.make_torch(n, dt, "uniform", device="cuda")
y = S.scan(x, k, s, True); torch.cuda.synchronize()
if n <= (1 << 22):
    ref = oracle.scan(x.cpu().numpy(), k, s, True)[0]
    got = y.cpu().numpy()
    ok = np.array_equal(got.view(ref.dtype), ref) if dt in ("i32", "i64") else np.allclose(got, ref, rtol=1e-3, atol=1e-3)
    print("OK" if ok else "MISMATCH")
else:
    print("RAN")
'''
for c in cfgs:
    dt, n, k, s = c.split(":")
    try:
        r = subprocess.run([sys.executable, "-c", code, dt, n, k, s], capture_output=True, text=True, timeout=60)
        out = (r.stdout.strip().splitlines() or [""])[-1] + " " + (r.stderr.strip().splitlines() or [""])[-1][:120]
    except subprocess.TimeoutExpired:
        out = "TIMEOUT (hang)"
    print(f"{c}: {out}", flush=True)
