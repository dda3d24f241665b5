"""Measure the delta ENCODER (sam_delta_encode) and the encode -> decode
round trip on one GPU.  One JSON line per (dtype, order, tuple):

    python tools/bench_delta.py [--reps 20] [--cases i32:1:1,i32:2:1,...]

Kernel time = CUDA events on the launching stream around `reps` back-to-back launches (inputs of
4 GiB per array > 126 MB L2, so no flush is needed); algorithmic bytes = 2 w n per launch (read x
once, write the differences once); peak = MEASURED_PEAKS.json hbm_gbs.  Round trip = encode + the
inclusive order-k scan (sam_scan), checked bit-exact (ints) after timing.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402

W = {"i32": 4, "i64": 8, "f32": 4, "f64": 8}


def timed(fn, reps):
    st = torch.cuda.current_stream()
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(reps):
        fn()
    e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--cases", default="i32:1:1,i32:2:1,i32:4:1,i32:8:1,i32:1:4,i32:3:8,i64:1:1,i64:4:4,"
                                       "i64:8:8,f32:2:3,f64:2:2")
    args = ap.parse_args()
    with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
        peak = float(json.load(f)["hbm_gbs"])
    for case in args.cases.split(","):
        name, k, s = case.split(":")
        k, s = int(k), int(s)
        n = (1 << 32) // W[name]  # 4 GiB per array
        x = synth.make_torch(n, name, "uniform", seed=11, device="cuda")
        d = torch.empty_like(x)
        y = torch.empty_like(x)
        mc = torch.empty_like(x)
        t_enc = timed(lambda: S.delta_encode(x, k, s, out=d), args.reps)
        t_mc = timed(lambda: mc.copy_(x), args.reps)
        t_rt = timed(lambda: (S.delta_encode(x, k, s, out=d), S.scan(d, k, s, True, out=y)), args.reps)
        ok = bool(torch.equal(y, x)) if name in ("i32", "i64") else None
        b = 2 * W[name] * n
        print(json.dumps({
            "kernel": "sam::delta_kernel", "dtype": name, "order": k, "tuple": s, "n": n,
            "encode_ms": t_enc, "encode_gbs": b / t_enc / 1e6, "encode_gvalues_s": n / t_enc / 1e6,
            "memcpy_gbs": b / t_mc / 1e6, "frac_of_memcpy": t_mc / t_enc,
            "roofline": {"bound": "hbm", "achieved": b / t_enc / 1e6, "peak": peak, "frac": b / t_enc / 1e6 / peak},
            "round_trip_ms": t_rt, "round_trip_gvalues_s": n / t_rt / 1e6, "round_trip_exact": ok,
        }), flush=True)
        del x, d, y, mc
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
