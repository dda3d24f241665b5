import sys, os, ctypes
sys.path.insert(0, "/root/repo")
import numpy as np, torch, oracle, synth
import paper_conf_pldi_malekiyb16_b200 as S
from paper_conf_pldi_malekiyb16_b200.dist import scan_cyclic_virtual, _cyclic_steps
for la in (0, 1):
    for (name, k, s) in (("i32", 1, 1), ("i32", 2, 1), ("i64", 2, 1), ("i32", 3, 3)):
        n, C = 200003, 7777
        x = synth.make(n, name, "uniform", seed=5)
        y = scan_cyclic_virtual(torch.from_numpy(x).cuda(), 1, C, k, s, True, lookahead=la)
        torch.cuda.synchronize()
        ref = oracle.scan(x, k, s, True)[0]
        yy = y.cpu().numpy().view(ref.dtype)
        bad = np.nonzero(yy != ref)[0]
        print(la, name, k, s, "bad", bad.size, bad[:3])
# manual p=1 driver with seeds printed
name, k, s, n, C = "i32", 2, 1, 40000, 7777
x = synth.make(n, name, "uniform", seed=5)
xt = torch.from_numpy(x).cuda(); out = torch.empty_like(xt)
gen = _cyclic_steps(xt, out, k, s, True, C, n, 0, 1, 0, torch.cuda.current_stream())
msg = next(gen); r = 0
import itertools
while True:
    try:
        if msg[0] == "send":
            pl = msg[2].clone(); torch.cuda.synchronize()
            st = pl.cpu().numpy()[16:16 + 4 * k * s].view(np.uint32)
            g0 = msg[1] * C
            _, run = oracle.scan(x[g0:g0 + C], k, s, True)
            print("send", msg[1], "payload", st, "oracle", run.reshape(-1), "hdr", pl.cpu().numpy()[:16].view(np.uint64))
            msg = gen.send(None)
        else:
            msg = gen.send(pl)
    except StopIteration:
        break
torch.cuda.synchronize()
ref = oracle.scan(x, k, s, True)[0]
yy = out.cpu().numpy().view(ref.dtype)
print("manual bad", np.nonzero(yy != ref)[0][:5])
