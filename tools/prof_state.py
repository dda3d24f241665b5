"""Run the state pass (sam_shard_state) a few times on one config (for ncu): python tools/prof_state.py i64 30 4 4"""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_pldi_malekiyb16_b200 as S
dt, logn, k, s = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
x = synth.make_torch(1 << logn, dt, "uniform", device="cuda")
dc = S.dtype_code(x.dtype)
pay = torch.zeros(S.sam_shard_payload_bytes(dc, k, s), dtype=torch.uint8, device="cuda")
for _ in range(3):
    S.sam_shard_state(dc, k, s, ctypes.c_void_p(x.data_ptr()), x.numel(), 0, ctypes.c_void_p(pay.data_ptr()))
torch.cuda.synchronize()
print("done")
