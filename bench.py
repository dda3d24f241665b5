#!/usr/bin/env python3
"""Benchmark of the SAM single-pass scan on B200 (BASELINE.json metric: Gvalues/s & HBM GB/s vs memcpy).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl {sam,reference}] [--config C2]

Workload (BASELINE.json configs[1], "C2"): n = 2^30 int32, order 1, tuple 1, inclusive, one B200.
A step is one pass of the whole hot path over one batch: one sam_scan launch (N = 1), or, under
torchrun with N > 1 ranks (weak scaling, 2^30 elements per GPU, contiguous shards of one global
array): sam_shard_state -> NCCL all_gather of the carry payloads -> sam_shard_scan.
Inputs (4 GiB per GPU) are larger than the 126 MB L2, so no L2 flush is needed between steps.

One JSON line is printed by rank 0.  `value` is whole-job Gvalues/s with inputs resident in HBM;
`e2e` is the same metric through the host-buffer C-ABI entry (sam_scan_host: pinned host input,
chunked H2D | scan | D2H pipeline, result back in host memory); `roofline` relates the scan
kernel's algorithmic bytes (2 x 4 B per element: one read + one write) to the measured
HBM copy peak; `cpu_baseline` is the CPU oracle (oracle/, serial, 1 core) on a bounded sample.

--impl reference times the oracle itself (the tier's reference arm) on the same config.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    # name: (dtype, log2 n, order, tuple, inclusive, description)
    "C1": ("i32", 20, 1, 1, True, "C1: n=2^20 int32 order-1 tuple-1 inclusive scan (L2-resident)"),
    "C2": ("i32", 30, 1, 1, True, "C2: n=2^30 int32 order-1 tuple-1 inclusive scan vs cudaMemcpy"),
    "C3k8": ("i32", 28, 8, 1, True, "C3: n=2^28 int32 order-8 tuple-1 inclusive scan"),
    "C3i64k8": ("i64", 28, 8, 1, True, "C3: n=2^28 int64 order-8 tuple-1 inclusive scan"),
    "C4s8": ("i64", 28, 1, 8, True, "C4: n=2^28 int64 order-1 tuple-8 inclusive scan"),
    "C5": ("i64", 30, 4, 4, True, "C5: int64 order-4 tuple-4 inclusive scan, 2^30 per GPU"),
    # the encoder, not the north-star path: --config D2 / D2k8
    "D2": ("i32", 30, 1, 1, True, "D2: n=2^30 int32 order-1 tuple-1 delta ENCODE (sam_delta_encode, NEXT-2)"),
    "D2k8": ("i32", 30, 8, 1, True, "D2k8: n=2^30 int32 order-8 tuple-1 delta ENCODE (sam_delta_encode, NEXT-2)"),
}


def is_delta(config_name):
    return config_name.startswith("D")
W_BYTES = {"i32": 4, "i64": 8, "f32": 4, "f64": 8}
DTYPE_NAME = {"i32": "int32", "i64": "int64", "f32": "float32", "f64": "float64"}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def ncu_traffic(config_name):
    """DRAM bytes per launch of the scan kernel from a committed ncu --set full capture, or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(config_name)
    return None


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 100 ms while the GPU is loaded."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index=0):
        self.gpu = gpu_index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
        return self

    def __exit__(self, *a):
        self.lines = []
        if self.proc is not None:
            self.proc.terminate()
            try:
                out, _ = self.proc.communicate(timeout=5)
            except Exception:
                self.proc.kill()
                out = ""
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        sm, mx, reasons, watts = [], None, set(), []
        for l in getattr(self, "lines", []):
            f = [x.strip() for x in l.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
                watts.append(float(f[3]))
            except ValueError:
                continue
            for name, val in zip(("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"), f[5:9]):
                if val.lower().startswith("active"):
                    reasons.add(name)
        loaded = [x for x, w in zip(sm, watts) if w > 250] or sm
        lw = [w for w in watts if w > 250] or watts
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm), "samples_under_load": len(loaded),
                "power_w": statistics.median(lw) if lw else None}


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform

    return platform.processor() or platform.machine()


# Every BASELINE.json config, one line each in the `sweep` key: name, dtype,
# log2 n, order, tuple.  C3: int32/int64 orders 1..8; C4: int64 tuples 1..8 at orders 1, 2 and
# fp32/fp64 tuples at order 1; C5: int64 order 4 tuple 4 at 2^30 (one GPU's weak-scaling share) and
# at 2^33 (the strong-scaling total, > 2^32 elements, 128 GiB of HBM).
SWEEP = ([("C1 i32 k=1 s=1 n=2^20 (L2-resident, launch-bound)", "i32", 20, 1, 1)] +
         [(f"C3 i32 k={k}", "i32", 28, k, 1) for k in range(1, 9)] +
         [(f"C3 i64 k={k}", "i64", 28, k, 1) for k in range(1, 9)] +
         [(f"C4 i64 k={k} s={s}", "i64", 28, k, s) for k in (1, 2) for s in range(1, 9)] +
         [(f"C4 {d} k=1 s={s}", d, 28, 1, s) for d in ("f32", "f64") for s in range(1, 9)] +
         [("C5 i64 k=4 s=4 n=2^30", "i64", 30, 4, 4), ("C5 i64 k=4 s=4 n=2^33", "i64", 33, 4, 4)])


def run_sweep(sam, synth, torch, peak, reps=5):
    """Kernel-only throughput of every config (CUDA events on the launching stream, inputs in HBM,
    > L2), against a memcpy of the same bytes and the measured copy peak."""
    import ctypes

    out = []
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    memcpy_cache = {}
    for name, dt, logn, k, s in SWEEP:
        n = 1 << logn
        w = W_BYTES[dt]
        free, _ = torch.cuda.mem_get_info()
        if free < 2 * n * w + (2 << 30):
            out.append({"config": name, "skipped": f"needs {2 * n * w / 2**30:.0f} GiB free HBM"})
            continue
        x = synth.make_torch(n, dt, "uniform" if dt[0] == "i" else "unif01", seed=synth.SEED_BASE + 2, device="cuda")
        y = torch.empty_like(x)
        st = torch.cuda.current_stream()
        sp = ctypes.c_void_p(st.cuda_stream)
        dc = sam.dtype_code(x.dtype)
        P = lambda t: ctypes.c_void_p(t.data_ptr())
        for _ in range(2):
            sam.sam_scan(dc, k, s, True, P(x), P(y), n, sp)
        torch.cuda.synchronize()
        e0.record(st)
        for _ in range(reps):
            sam.sam_scan(dc, k, s, True, P(x), P(y), n, sp)
        e1.record(st)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        key = (n, w)
        if key not in memcpy_cache:
            for _ in range(2):
                y.copy_(x)
            e0.record(st)
            for _ in range(reps):
                y.copy_(x)
            e1.record(st)
            torch.cuda.synchronize()
            memcpy_cache[key] = e0.elapsed_time(e1) / reps
        gbs = 2 * w * n / (ms * 1e-3) / 1e9
        if logn <= 24:  # L2-resident: also the exclusive scan, and the per-launch time (launch-bound)
            e0.record(st)
            for _ in range(reps):
                sam.sam_scan(dc, k, s, False, P(x), P(y), n, sp)
            e1.record(st)
            torch.cuda.synchronize()
            out.append({"config": name + " exclusive", "n": n, "order": k, "tuple": s, "dtype": DTYPE_NAME[dt],
                        "us_per_launch": e0.elapsed_time(e1) / reps * 1e3,
                        "gvalues_s": n / (e0.elapsed_time(e1) / reps * 1e-3) / 1e9, "l2_resident": True})
        out.append({"config": name, "n": n, "order": k, "tuple": s, "dtype": DTYPE_NAME[dt],
                    "gvalues_s": n / (ms * 1e-3) / 1e9, "gbs": gbs, "ms": ms,
                    "frac_of_memcpy": memcpy_cache[key] / ms, "roofline_frac": gbs / peak,
                    "traffic": ncu_traffic(name)})
        del x, y
        torch.cuda.empty_cache()
    return out


def time_sharded(sam, synth, torch, dist, dt, n_local, k, s, rank, world, local, reps=5):
    """One sharded step (sam_shard_state -> NCCL all-gather of the payloads -> sam_shard_scan) on
    n_local elements per rank, CUDA events on the launching stream, max over ranks; plus the state
    pass alone (its cost relative to the scan: the reduce-then-scan overhead)."""
    import ctypes

    free, _ = torch.cuda.mem_get_info()
    w = W_BYTES[dt]
    if free < 2 * n_local * w + (3 << 30):
        return {"skipped": f"needs {2 * n_local * w / 2**30:.0f} GiB free HBM per GPU"}
    g_off = rank * n_local
    x = synth.make_torch(n_local, dt, "uniform", seed=synth.SEED_BASE + 5, start=g_off, device=torch.device("cuda", local))
    y = torch.empty_like(x)
    dc = sam.dtype_code(x.dtype)
    st = torch.cuda.current_stream()
    sp = ctypes.c_void_p(st.cuda_stream)
    P = lambda t: ctypes.c_void_p(t.data_ptr())
    pb = sam.sam_shard_payload_bytes(dc, k, s)
    payload = torch.empty(pb, dtype=torch.uint8, device=x.device)
    gathered = torch.empty(world * pb, dtype=torch.uint8, device=x.device)

    def state():
        sam.sam_shard_state(dc, k, s, P(x), n_local, g_off, P(payload), sp)

    def step():
        state()
        if world > 1:
            dist.all_gather_into_tensor(gathered, payload)
        else:
            gathered.copy_(payload)
        sam.sam_shard_scan(dc, k, s, True, P(x), P(y), n_local, g_off, P(gathered), rank, world, sp)

    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    res = {}
    for name, fn in (("step", step), ("state", state)):
        for _ in range(2):
            fn()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        e0.record(st)
        for _ in range(reps):
            fn()
        e1.record(st)
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1) / reps], dtype=torch.float64, device=x.device)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        res[name + "_ms"] = float(t[0])
    n_total = n_local * world
    res.update({"n_per_gpu": n_local, "n_total": n_total, "order": k, "tuple": s, "dtype": DTYPE_NAME[dt],
                "gvalues_s": n_total / (res["step_ms"] * 1e-3) / 1e9,
                "per_gpu_hbm_gbs_algorithmic": 2 * w * n_local / (res["step_ms"] * 1e-3) / 1e9,
                "state_over_step": res["state_ms"] / res["step_ms"]})
    del x, y
    torch.cuda.empty_cache()
    return res


def time_cyclic(sam, synth, torch, dist, dt, n_local, k, s, rank, world, local, chunk=1 << 24, reps=3):
    """One block-cyclic step (NEXT-1: per round a state pass over this rank's chunk, an all-gather of
    the round's payloads, sam_cyclic_fold, the seeded scan of the chunk), max over ranks."""
    from paper_conf_pldi_malekiyb16_b200.dist import cyclic_local_len, scan_cyclic, scan_cyclic_virtual

    free, _ = torch.cuda.mem_get_info()
    w = W_BYTES[dt]
    if free < 2 * n_local * w + (3 << 30):
        return {"skipped": f"needs {2 * n_local * w / 2**30:.0f} GiB free HBM per GPU"}
    n_total = n_local * world
    nl = cyclic_local_len(n_total, chunk, world, rank)
    x = synth.make_torch(nl, dt, "uniform", seed=synth.SEED_BASE + 9, device=torch.device("cuda", local))
    y = torch.empty_like(x)
    st = torch.cuda.current_stream()
    if world > 1:
        fn = lambda: scan_cyclic(x, k, s, True, chunk=chunk, n_total=n_total, out=y)
    else:
        fn = lambda: scan_cyclic_virtual(x, 1, chunk, k, s, True, lookahead=0)
    fn()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(reps):
        fn()
    e1.record(st)
    torch.cuda.synchronize()
    t = torch.tensor([e0.elapsed_time(e1) / reps], dtype=torch.float64, device=x.device)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t[0])
    del x, y
    torch.cuda.empty_cache()
    return {"chunk": chunk, "step_ms": ms, "n_per_gpu": n_local, "n_total": n_total, "order": k, "tuple": s,
            "dtype": DTYPE_NAME[dt], "gvalues_s": n_total / (ms * 1e-3) / 1e9,
            "rounds": -(-(-(-n_total // chunk)) // world)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def run_reference(args):
    """Reference arm: the CPU oracle (serial, 1 core) on the same config, bounded sample per step."""
    world, rank, _ = dist_env()
    if rank != 0:
        return 0
    import numpy as np

    import oracle
    import synth

    dt, logn, k, s, incl, desc = CONFIGS[args.config]
    n_total = (1 << logn) * max(1, args.gpus)
    sample = min(n_total, 1 << 27)  # bounded: ~0.1-1 s of serial CPU work per step
    x = synth.make(sample, dt, "uniform", seed=synth.SEED_BASE + 1)
    run = (lambda a: oracle.delta(a, k, s)) if is_delta(args.config) else (lambda a: oracle.scan(a, k, s, incl))
    run(x[: 1 << 16])
    for _ in range(args.warmup):
        run(x[: 1 << 20])
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        run(x)
        times.append(time.perf_counter() - t0)
    t = statistics.median(times)
    gv = sample / t / 1e9
    line = {
        "impl": "reference", "metric": "Gvalues/s", "value": gv, "unit": "Gvalues/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": DTYPE_NAME[dt], "data": "synthetic",
        "config": {"workload": desc, "n": n_total, "order": k, "tuple": s, "inclusive": incl},
        "cpu_baseline": {"value": gv, "unit": "Gvalues/s", "cores": 1, "kind": "oracle",
                         "sample": f"first {sample} elements of the workload, serial oracle loop, median of {args.steps}"},
        "e2e": {"value": gv, "unit": "Gvalues/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="sam", choices=["sam", "reference"])
    ap.add_argument("--config", default="C2", choices=sorted(CONFIGS))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-sweep", action="store_true", help="skip the per-config sweep (C3/C4/C5) key")
    ap.add_argument("--cyclic", action="store_true", help="also time the block-cyclic path at N=1 (always at N>1)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_pldi_malekiyb16_b200 as sam
    import synth
    from paper_conf_pldi_malekiyb16_b200.dist import exchange_payloads

    world, rank, local = dist_env()
    if world > 1:
        dist.init_process_group("nccl")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dt, logn, k, s, incl, desc = CONFIGS[args.config]
    w = W_BYTES[dt]
    n_local = 1 << logn
    g_off = rank * n_local
    x = synth.make_torch(n_local, dt, "uniform", seed=synth.SEED_BASE + 1, start=g_off, device=dev)
    y = torch.empty_like(x)
    dc = sam.dtype_code(x.dtype)
    stream = torch.cuda.current_stream()
    sp = sam._stream_ptr(stream)
    import ctypes

    P = lambda t, off=0: ctypes.c_void_p(t.data_ptr() + off)
    pb = sam.sam_shard_payload_bytes(dc, k, s)
    payload = torch.empty(pb, dtype=torch.uint8, device=dev)
    gathered = torch.empty(world * pb, dtype=torch.uint8, device=dev)
    ev_k0 = torch.cuda.Event(enable_timing=True)
    ev_k1 = torch.cuda.Event(enable_timing=True)
    kern_ms = []

    delta = is_delta(args.config)
    if delta and world > 1:
        from paper_conf_pldi_malekiyb16_b200.dist import delta_encode_sharded

    def step(time_kernel=False):
        if delta:
            if time_kernel:
                ev_k0.record(stream)
            if world == 1:
                sam.sam_delta_encode(dc, k, s, P(x), P(y), n_local, sp)
            else:
                delta_encode_sharded(x, k, s, out=y)
            if time_kernel:
                ev_k1.record(stream)
        elif world == 1:
            if time_kernel:
                ev_k0.record(stream)
            sam.sam_scan(dc, k, s, incl, P(x), P(y), n_local, sp)
            if time_kernel:
                ev_k1.record(stream)
        else:
            sam.sam_shard_state(dc, k, s, P(x), n_local, g_off, P(payload), sp)
            dist.all_gather_into_tensor(gathered, payload)
            if time_kernel:
                ev_k0.record(stream)
            sam.sam_shard_scan(dc, k, s, incl, P(x), P(y), n_local, g_off, P(gathered), rank, world, sp)
            if time_kernel:
                ev_k1.record(stream)

    # warm-up (and a short clock soak so the timed region sees steady clocks)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t_soak = time.perf_counter()
        while time.perf_counter() - t_soak < 0.6:
            step()
        torch.cuda.synchronize()
        # ---- timed region ----
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        launches0 = sam.sam_launch_count()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        launches = sam.sam_launch_count() - launches0
        elapsed = e0.elapsed_time(e1)  # ms
        # scan-kernel-only timing (same stream, same launches, separate pass) for the roofline
        for _ in range(args.steps):
            step(time_kernel=True)
            torch.cuda.synchronize()
            kern_ms.append(ev_k0.elapsed_time(ev_k1))
    t = torch.tensor([elapsed, statistics.mean(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    elapsed, kavg = float(t[0]), float(t[1])
    ms_per_step = elapsed / args.steps
    n_total = n_local * world
    value = n_total / (ms_per_step * 1e-3) / 1e9

    # memcpy of the same bytes (context: SAM's target is memcpy speed)
    mc = torch.empty_like(x)
    for _ in range(3):
        mc.copy_(x)
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(10):
        mc.copy_(x)
    e1.record(stream)
    torch.cuda.synchronize()
    memcpy_ms = e0.elapsed_time(e1) / 10
    del mc

    # correctness spot check of the timed output against the oracle on a prefix (not timed)
    check = None
    if rank == 0 and world == 1:
        import oracle

        m = 1 << 20
        ref = oracle.delta(x[:m].cpu().numpy(), k, s) if delta else oracle.scan(x[:m].cpu().numpy(), k, s, incl)[0]
        got = y[:m].cpu().numpy().view(ref.dtype)
        check = bool(np.array_equal(got, ref))

    # end-to-end through the host-buffer C-ABI entry (pinned memory, H2D | scan | D2H pipeline)
    e2e = None
    if not args.no_e2e:
        xh = x.cpu().pin_memory()
        yh = torch.empty_like(xh).pin_memory()
        if delta and world == 1:
            sam.sam_delta_encode_host(dc, k, s, P(xh), P(yh), n_local, sp)
            tt = []
            for _ in range(3):
                t0 = time.perf_counter()
                sam.sam_delta_encode_host(dc, k, s, P(xh), P(yh), n_local, sp)
                tt.append(time.perf_counter() - t0)
            te = statistics.median(tt)
        elif delta:
            # encoder e2e under torchrun: pinned H2D, halo-exchanged encode, D2H
            xd = torch.empty_like(x)
            yd = torch.empty_like(x)
            tt = []
            for _ in range(4):
                dist.barrier()
                t0 = time.perf_counter()
                xd.copy_(xh, non_blocking=True)
                delta_encode_sharded(xd, k, s, out=yd)
                yh.copy_(yd, non_blocking=True)
                torch.cuda.synchronize()
                tt.append(time.perf_counter() - t0)
            tte = torch.tensor([statistics.median(tt[1:])], dtype=torch.float64, device=dev)
            dist.all_reduce(tte, op=dist.ReduceOp.MAX)
            te = float(tte[0])
            del xd, yd
        elif world == 1:
            sam.sam_scan_host(dc, k, s, incl, P(xh), P(yh), n_local, sp)
            reps = 3
            tt = []
            for _ in range(reps):
                t0 = time.perf_counter()
                sam.sam_scan_host(dc, k, s, incl, P(xh), P(yh), n_local, sp)
                tt.append(time.perf_counter() - t0)
            te = statistics.median(tt)
        else:
            xd = torch.empty_like(x)
            yd = torch.empty_like(x)
            tt = []
            for _ in range(3):
                dist.barrier()
                t0 = time.perf_counter()
                xd.copy_(xh, non_blocking=True)
                sam.sam_shard_state(dc, k, s, P(xd), n_local, g_off, P(payload), sp)
                dist.all_gather_into_tensor(gathered, payload)
                sam.sam_shard_scan(dc, k, s, incl, P(xd), P(yd), n_local, g_off, P(gathered), rank, world, sp)
                yh.copy_(yd, non_blocking=True)
                torch.cuda.synchronize()
                tt.append(time.perf_counter() - t0)
            tte = torch.tensor([statistics.median(tt)], dtype=torch.float64, device=dev)
            dist.all_reduce(tte, op=dist.ReduceOp.MAX)
            te = float(tte[0])
        e2e = {"value": n_total / te / 1e9, "unit": "Gvalues/s", "h2d_bytes_per_step": n_local * w * world,
               "d2h_bytes_per_step": n_local * w * world, "ms_per_step": te * 1e3,
               "path": "sam_delta_encode_host: pinned host buffers, 128 MiB chunks, H2D | encode | D2H on 3 streams"
               if delta and world == 1 else "per rank: pinned H2D, tail all-gather, encode, D2H" if delta else
               "sam_scan_host: pinned host buffers, 128 MiB chunks, H2D | seeded scan | D2H on 3 streams"
               if world == 1 else "per rank: pinned H2D, shard state, NCCL all-gather, shard scan, D2H"}

    # CPU oracle baseline on a bounded sample of the same workload (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        import oracle

        sample = 1 << 27
        xs = x[:sample].cpu().numpy()
        orun = (lambda a: oracle.delta(a, k, s)) if delta else (lambda a: oracle.scan(a, k, s, incl))
        orun(xs[: 1 << 20])
        ts = []
        for _ in range(3):
            t0 = time.perf_counter()
            orun(xs)
            ts.append(time.perf_counter() - t0)
        cpu = {"value": sample / statistics.median(ts) / 1e9, "unit": "Gvalues/s", "cores": 1, "kind": "oracle",
               "sample": f"first 2^27 elements of the same input, serial oracle (oracle/sam_oracle.c), median of 3",
               "cpu_model": cpu_model(), "nproc": os.cpu_count()}
        if dt in ("i32", "i64") and not delta and incl:
            # context only: all host cores, k passes of two-phase order-1 scans (oracle/cpu_allcores.c)
            nt = os.cpu_count() or 1
            oracle.scan_allcores(xs[: 1 << 20], k, s, threads=nt)
            ta = []
            for _ in range(3):
                t0 = time.perf_counter()
                oracle.scan_allcores(xs, k, s, threads=nt)
                ta.append(time.perf_counter() - t0)
            cpu["allcores"] = {"value": sample / statistics.median(ta) / 1e9, "unit": "Gvalues/s", "threads": nt,
                               "kind": "all-cores context scan (k passes of two-phase order-1 scans, OpenMP)",
                               "sample": "same 2^27-element sample, median of 3"}

    peak, peak_src = measured_peaks()
    sweep = None
    sharded = None
    if not args.no_sweep and not delta:
        del y
        torch.cuda.empty_cache()
        if world == 1:
            sweep = run_sweep(sam, synth, torch, peak)
        # north_star's multi-GPU config C5 (int64, order 4, tuple 4): weak (2^30 per GPU) and strong
        # (2^33 in total) through the sharded path, max over ranks; and the state pass alone (K*2)
        sharded = {}
        for tag, nl in (("c5_weak", 1 << 30), ("c5_strong", (1 << 33) // world)):
            sharded[tag] = time_sharded(sam, synth, torch, dist, "i64", nl, 4, 4, rank, world, local)
        if world > 1 or args.cyclic:  # NEXT-1: the block-cyclic layout, C5 weak
            sharded["cyclic_c5_weak"] = time_cyclic(sam, synth, torch, dist, "i64", 1 << 30, 4, 4, rank, world, local)
    alg_bytes = 2 * w * n_local
    achieved = alg_bytes / (kavg * 1e-3) / 1e9
    if rank == 0:
        line = {
            "metric": "Gvalues/s", "value": value, "unit": "Gvalues/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": DTYPE_NAME[dt], "data": "synthetic",
            "config": {"workload": desc, "n_per_gpu": n_local, "n_total": n_total, "order": k, "tuple": s,
                       "inclusive": incl, "input": "splitmix64 uniform (synth/), generated in HBM",
                       "l2": f"inputs {n_local * w / 2**30:.1f} GiB per GPU > 126 MB L2: no flush needed",
                       "parallelism": "single GPU" if world == 1 else
                       f"{world} contiguous shards, NCCL all_gather of {pb}-B carry payloads"},
            "hbm_gbs": alg_bytes / (ms_per_step * 1e-3) / 1e9,
            "memcpy_gbs": 2 * w * n_local / (memcpy_ms * 1e-3) / 1e9,
            "frac_of_memcpy": memcpy_ms / ms_per_step,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": ncu_traffic(args.config),
                         "kernel": "sam::delta_kernel" if delta else "sam::sam_scan_kernel", "kernel_ms": kavg,
                         "algorithmic_bytes_per_launch": alg_bytes, "peak_source": peak_src},
            "cpu_baseline": cpu,
            "sweep": sweep,
            "sharded_c5": sharded,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk.summary(),
            "parity_prefix_check": check,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
