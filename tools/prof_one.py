"""Run one scan config a few times (for ncu: profile the last launch)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
dt, logn, k, s = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 3
x = synth.make_torch(1 << logn, dt, "uniform", device="cuda")
y = torch.empty_like(x)
for _ in range(reps):
    S.scan(x, k, s, True, out=y)
torch.cuda.synchronize()
print("done", dt, logn, k, s)
