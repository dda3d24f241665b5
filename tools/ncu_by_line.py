"""Aggregate an ncu source page (--print-source cuda,sass) by CUDA source line (developer tool).
    ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > X.csv; python tools/ncu_by_line.py X.csv [top]"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
agg = collections.defaultdict(lambda: [0.0, 0.0, ""])
fname = ""
hdr = None
for r in rows:
    if not r: continue
    if r[0] == "File Path": fname = r[1].split("/")[-1]; continue
    if r[0] == "Line No": hdr = r; continue
    if hdr is None or r[0] in ("Function Name",): continue
    if len(r) < 8: continue
    try: line = int(r[0])
    except ValueError: continue
    i_s = hdr.index("Warp Stall Sampling (All Samples)"); i_e = hdr.index("Instructions Executed")
    try:
        st = float(r[i_s] or 0); ex = float(r[i_e] or 0)
    except ValueError: continue
    a = agg[(fname, line)]; a[0] += st; a[1] += ex; a[2] = r[1][:90]
ts = sum(v[0] for v in agg.values()) or 1; te = sum(v[1] for v in agg.values()) or 1
print(f"total samples {ts:.0f}, warp-instructions {te:.3e}")
for (f, l), (st, ex, src) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{st/ts*100:5.1f}% stall  {ex/te*100:5.1f}% inst  {f}:{l:<5} {src}")
