import sys, os, ctypes
sys.path.insert(0, "/root/repo")
import numpy as np, torch, oracle, synth
import paper_conf_pldi_malekiyb16_b200 as S
name, k, s, n, C = "i32", 2, 1, 40000, 7777
x = synth.make(n, name, "uniform", seed=5)
xt = torch.from_numpy(x).cuda(); out = torch.empty_like(xt)
P = lambda t, off=0: ctypes.c_void_p(t.data_ptr() + off)
pb = S.sam_shard_payload_bytes(0, k, s)
base = torch.zeros(k * s, dtype=torch.int32, device="cuda"); seedbuf = torch.empty_like(base)
for r in range(6):
    g0 = r * C; ln = min(C, n - g0)
    pay = torch.empty(pb, dtype=torch.uint8, device="cuda")
    S.sam_shard_state(0, k, s, P(xt, 4 * g0), ln, g0, P(pay))
    S.sam_cyclic_fold(0, k, s, P(pay), 0, 1, P(base), P(seedbuf), P(base))
    torch.cuda.synchronize()
    _, run = oracle.scan(x[:g0], k, s, True)
    _, run2 = oracle.scan(x[:g0 + ln], k, s, True)
    print(r, "seed", seedbuf.cpu().numpy().view(np.uint32), "oracle", run.reshape(-1), "base", base.cpu().numpy().view(np.uint32), run2.reshape(-1))
    S.sam_scan_seeded(0, k, s, 1, P(xt, 4 * g0), P(out, 4 * g0), ln, g0, P(seedbuf), None)
torch.cuda.synchronize()
ref = oracle.scan(x, k, s, True)[0]
print("bad", np.nonzero(out.cpu().numpy().view(np.uint32) != ref)[0][:5])
