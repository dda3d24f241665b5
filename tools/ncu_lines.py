"""Top CUDA source lines by warp-stall samples from an .ncu-rep (developer tool): python tools/ncu_lines.py rep [top]"""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass,cuda"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = next(i for i, r in enumerate(rows) if "Warp Stall Sampling (All Samples)" in r)
hdr = rows[h]; data = [r for r in rows[h + 1:] if len(r) == len(hdr)]
i_s = hdr.index("Warp Stall Sampling (All Samples)")
agg = defaultdict(float); src = {}
for r in data:
    try:
        v = float(r[i_s] or 0)
    except ValueError:
        continue
    agg[r[0]] += v; src[r[0]] = r[1]
tot = sum(agg.values()) or 1
for ln, v in sorted(agg.items(), key=lambda x: -x[1])[:top]:
    print(f"{v / tot * 100:5.1f}% L{ln:>5} {src[ln].strip()[:110]}")
