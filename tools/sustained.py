"""Sustained (power-capped) throughput of one config (developer tool): 1 s soak, then K timed
launches, with the nvidia-smi clock/power sampler of bench.py.
    python tools/sustained.py i32 30 1 1 [K]     (SAM_LIB_PATH selects a library variant)"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402
from bench import ClockSampler  # noqa: E402

dt, logn, k, s = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
K = int(sys.argv[5]) if len(sys.argv) > 5 else 50
n = 1 << logn
x = synth.make_torch(n, dt, "uniform", device="cuda")
y = torch.empty_like(x)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
with ClockSampler(0) as clk:
    t0 = time.time()
    while time.time() - t0 < 1.0:
        S.scan(x, k, s, True, out=y)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(K):
        S.scan(x, k, s, True, out=y)
    e1.record()
    torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / K
print(json.dumps({"lib": os.environ.get("SAM_LIB_PATH", "default"), "config": f"{dt} 2^{logn} k={k} s={s}",
                  "gbs": 2 * n * x.element_size() / (ms * 1e-3) / 1e9, "ms": ms, "clocks": clk.summary()}), flush=True)
