"""Driver for tests/test_sanitizer_gpu.py: a few small scans through the C ABI, each checked against
the oracle, meant to run under compute-sanitizer (racecheck / synccheck / memcheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402


def main():
    bad = 0
    for name in ("i32", "i64"):
        for k in (1, 4, 8):
            for s in (1, 3, 8):
                n = 3 * 7168 + 1234
                xn = synth.make(n, name, "uniform", seed=k * 10 + s)
                x = torch.from_numpy(xn).cuda()
                for incl in (True, False):
                    y = S.scan(x, k, s, incl)
                    torch.cuda.synchronize()
                    ref = oracle.scan(xn, k, s, incl)[0]
                    if not np.array_equal(y.cpu().numpy().view(ref.dtype), ref):
                        print(f"MISMATCH {name} k={k} s={s} incl={incl}", flush=True)
                        bad += 1
    print("sanitize driver done, mismatches:", bad, flush=True)
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
