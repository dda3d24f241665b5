import sys, os, ctypes
sys.path.insert(0, "/root/repo")
import numpy as np, torch, oracle, synth
import paper_conf_pldi_malekiyb16_b200 as S
k, s, n, C = 2, 1, 20000, 7777
x = synth.make(n, "i32", "uniform", seed=5)
xt = torch.from_numpy(x).cuda()
pb = S.sam_shard_payload_bytes(0, k, s)
pay = torch.zeros(pb, dtype=torch.uint8, device="cuda")
P = lambda t, off=0: ctypes.c_void_p(t.data_ptr() + off)
S.sam_shard_state(0, k, s, P(xt), C, 0, P(pay))
torch.cuda.synchronize()
st = pay.cpu().numpy()[16:16 + 4 * k * s].view(np.uint32)
_, run = oracle.scan(x[:C], k, s, True)
print("payload", st, "oracle", run.reshape(-1))
base = torch.zeros(k * s, dtype=torch.int32, device="cuda"); seed = torch.zeros_like(base)
S.sam_cyclic_fold(0, k, s, P(pay), 0, 1, P(base), P(seed), P(base))
torch.cuda.synchronize()
print("seed", seed.cpu().numpy().view(np.uint32), "base", base.cpu().numpy().view(np.uint32))
base2 = torch.zeros_like(base)
S.sam_cyclic_fold(0, k, s, P(pay), 0, 1, None, P(seed), P(base2))
torch.cuda.synchronize()
print("seed(null base)", seed.cpu().numpy().view(np.uint32), "base2", base2.cpu().numpy().view(np.uint32))
out = torch.empty_like(xt)
S.sam_scan_seeded(0, k, s, 1, P(xt, 4 * C), P(out, 4 * C), C, C, P(base2), None)
torch.cuda.synchronize()
ref = oracle.scan(x[:2 * C], k, s, True)[0]
print("chunk1 ok", np.array_equal(out.cpu().numpy()[C:2 * C].view(np.uint32), ref[C:2 * C]))
# seeded continuation over a grid: chunk 0 -> final state -> chunk 1 seeded with it
bad = []
for name, dt, tdt, w in (("i32", 0, torch.int32, 4), ("i64", 1, torch.int64, 8)):
    for kk in range(1, 9):
        for ss in (1, 2, 3, 4, 8):
            for C1 in (7777, 8192, 100000):
                n2 = 2 * C1 + 5
                xx = synth.make(n2, name, "uniform", seed=kk * 10 + ss)
                xg = torch.from_numpy(xx).cuda(); yo = torch.empty_like(xg)
                stt = torch.zeros(kk * ss, dtype=tdt, device="cuda")
                S.sam_scan_seeded(dt, kk, ss, 1, P(xg), P(yo), C1, 0, None, P(stt))
                S.sam_scan_seeded(dt, kk, ss, 1, P(xg, w * C1), P(yo, w * C1), n2 - C1, C1, P(stt), None)
                torch.cuda.synchronize()
                ref = oracle.scan(xx, kk, ss, True)[0]
                if not np.array_equal(yo.cpu().numpy().view(ref.dtype), ref):
                    bad.append((name, kk, ss, C1))
print("seeded continuation failures:", bad)
