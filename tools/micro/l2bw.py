import ctypes, os, torch
L = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libl2bw.so"))
L.run_rd.restype = ctypes.c_float
L.run_rd.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p]
sink = torch.zeros(1, dtype=torch.int32, device="cuda")
for mb, iters in ((16, 200), (32, 100), (48, 100), (64, 60), (96, 40), (128, 30), (4096, 2)):
    x = torch.ones(mb << 18, dtype=torch.int32, device="cuda")
    ms = L.run_rd(x.data_ptr(), mb << 20, iters, sink.data_ptr())
    print(f"read {mb:5d} MB x{iters}: {mb * (1<<20) * iters / ms / 1e6:8.0f} GB/s", flush=True)
