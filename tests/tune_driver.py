"""Driver for tests/test_tune_gpu.py: runs in a fresh process with SAM_TUNE_FILE pointing at a table,
scans a few configs, checks each against the oracle and prints the launch shapes as JSON."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import oracle  # noqa: E402
import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402

out = {}
for name, k, s, n in (("i64", 2, 1, 3_000_011), ("i32", 4, 4, 5_000_003), ("i64", 1, 8, 1 << 20)):
    xn = synth.make(n, name, "uniform", seed=k * 8 + s)
    y = S.scan(torch.from_numpy(xn).cuda(), k, s, True)
    torch.cuda.synchronize()
    ok = bool(np.array_equal(y.cpu().numpy().view(np.uint64 if name == "i64" else np.uint32), oracle.scan(xn, k, s, True)[0]))
    out[f"{name} k={k} s={s}"] = dict(S.sam_debug_last_shape(), ok=ok)
print(json.dumps(out))
