"""Stall reasons and instruction counts by kernel region (developer tool).
    ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > X.csv
    python tools/ncu_regions.py X.csv name:lo-hi ...   (line ranges of sam_kernel.cuh)"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
regions = [(a.split(":")[0], *map(int, a.split(":")[1].split("-"))) for a in sys.argv[2:]]
hdr = None; fname = ""
tot = collections.defaultdict(lambda: collections.Counter())
for r in rows:
    if not r: continue
    if r[0] == "File Path" or r[0] == "File Name": fname = r[1]; continue
    if "Warp Stall Sampling (All Samples)" in r: hdr = r; continue
    if hdr is None or len(r) != len(hdr): continue
    try: line = int(r[0])
    except ValueError: continue
    reg = "other"
    if fname.endswith("sam_kernel.cuh"):
        for nm, lo, hi in regions:
            if lo <= line <= hi: reg = nm; break
    else:
        reg = "helpers"
    c = tot[reg]
    for i, h in enumerate(hdr):
        if h.startswith("stall_") and "Not Issued" not in h or h in ("Warp Stall Sampling (All Samples)", "Instructions Executed"):
            try: c[h] += float(r[i] or 0)
            except ValueError: pass
S = sum(c["Warp Stall Sampling (All Samples)"] for c in tot.values()) or 1
I = sum(c["Instructions Executed"] for c in tot.values()) or 1
for reg, c in sorted(tot.items(), key=lambda kv: -kv[1]["Warp Stall Sampling (All Samples)"]):
    st = c["Warp Stall Sampling (All Samples)"]
    top = sorted(((k[6:], v) for k, v in c.items() if k.startswith("stall_")), key=lambda kv: -kv[1])[:6]
    print(f"{reg:10s} samples {st/S*100:5.1f}%  inst {c['Instructions Executed']/I*100:5.1f}%  " +
          " ".join(f"{k}:{v/max(st,1)*100:.0f}%" for k, v in top))
