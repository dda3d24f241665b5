"""Run every bench.py sweep config twice (for an ncu DRAM-traffic pass; developer tool).
    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:sam_scan_kernel \\
        --csv --log-file gpurun_out/ncu_sweep.csv python tools/ncu_sweep.py
    python tools/ncu_sweep.py --parse gpurun_out/ncu_sweep.csv  -> profiles/ncu_traffic.json entries"""
import csv, json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

if len(sys.argv) > 2 and sys.argv[1] == "--parse":
    rows = [r for r in csv.reader(open(sys.argv[2])) if len(r) > 10]
    hdr = rows[0]
    iid, iname, ival = hdr.index("ID"), hdr.index("Metric Name"), hdr.index("Metric Value")
    per = {}
    for r in rows[1:]:
        per.setdefault(int(r[iid]), {})[r[iname]] = float(r[ival].replace(",", ""))
    ids = sorted(per)
    cfgs = [c for c in bench.SWEEP]
    out = {}
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    d = json.load(open(path)) if os.path.exists(path) else {}
    for j, c in enumerate(cfgs):
        if 2 * j + 1 >= len(ids):
            break
        m = per[ids[2 * j + 1]]
        d[c[0]] = m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]
        out[c[0]] = {"traffic": d[c[0]], "algorithmic": 2 * (1 << c[2]) * bench.W_BYTES[c[1]],
                     "ncu_ms": m["gpu__time_duration.sum"] / 1e6}
    d["_note_sweep"] = ("dram__bytes_read.sum + dram__bytes_write.sum of one sam_scan_kernel launch per sweep config "
                        "(ncu --metrics, clock-control none, second launch of each), tools/ncu_sweep.py")
    json.dump(d, open(path, "w"), indent=1)
    print(json.dumps(out, indent=1))
    sys.exit(0)

import ctypes  # noqa: E402
import torch  # noqa: E402
import paper_conf_pldi_malekiyb16_b200 as S  # noqa: E402
import synth  # noqa: E402

for name, dt, logn, k, s in bench.SWEEP:
    n = 1 << logn
    free, _ = torch.cuda.mem_get_info()
    if free < 2 * n * bench.W_BYTES[dt] + (2 << 30):
        print("skip", name)
        continue
    x = synth.make_torch(n, dt, "uniform" if dt[0] == "i" else "unif01", seed=synth.SEED_BASE + 2, device="cuda")
    y = torch.empty_like(x)
    for _ in range(2):
        S.scan(x, k, s, True, out=y)
    torch.cuda.synchronize()
    del x, y
    torch.cuda.empty_cache()
    print("done", name, flush=True)
