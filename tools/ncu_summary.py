"""Summarise an .ncu-rep: key metrics + top stall SASS lines (developer tool)."""
import csv, io, subprocess, sys

def details(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    r = csv.reader(io.StringIO(out)); hdr = next(r); rows = []
    for row in r:
        d = dict(zip(hdr, row)); rows.append((d.get("Section Name", ""), d.get("Metric Name", ""), d.get("Metric Unit", ""), d.get("Metric Value", "")))
    return rows

def raw(rep, names):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out))); hdr, units, vals = r[0], r[1], r[2]
    return {n: (vals[hdr.index(n)], units[hdr.index(n)]) for n in names if n in hdr}

def source(rep, top=25):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out))); hdr = rows[1]; data = rows[2:]
    i_s = hdr.index("Warp Stall Sampling (All Samples)"); i_e = hdr.index("Instructions Executed"); i_src = hdr.index("Source")
    tot = sum(float(r[i_s] or 0) for r in data) or 1
    res = []
    for r in sorted(data, key=lambda r: -float(r[i_s] or 0))[:top]:
        res.append(f"{float(r[i_s])/tot*100:5.1f}% {r[i_e]:>10} {r[i_src][:100]}")
    return res

if __name__ == "__main__":
    rep = sys.argv[1]
    keep = {"Duration", "DRAM Throughput", "Memory Throughput", "Registers Per Thread", "Achieved Occupancy", "Theoretical Occupancy",
            "Executed Ipc Active", "Issue Slots Busy", "L2 Hit Rate", "Dynamic Shared Memory Per Block", "Block Limit Registers",
            "Block Limit Shared Mem", "Executed Instructions", "Warp Cycles Per Issued Instruction", "Grid Size", "Block Size"}
    for sec, name, unit, val in details(rep):
        if name in keep: print(f"{name:40s} {val:>14} {unit}")
    for k, (v, u) in raw(rep, ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "lts__t_bytes.sum", "sm__inst_executed.sum"]).items():
        print(f"{k:40s} {v:>14} {u}")
    if "--src" in sys.argv:
        print("\n".join(source(rep)))

def stall_table(rep, top=20):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out))); hdr = rows[1]; data = rows[2:]
    cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    tot = {c: sum(float(r[hdr.index(c)] or 0) for r in data) for c in cols}
    T = sum(tot.values()) or 1
    print("stall totals:", ", ".join(f"{c[6:]}={v/T*100:.1f}%" for c, v in sorted(tot.items(), key=lambda x: -x[1]) if v / T > 0.005))
    i_s = hdr.index("Warp Stall Sampling (All Samples)"); i_src = hdr.index("Source"); i_a = hdr.index("Address")
    for r in sorted(data, key=lambda r: -float(r[i_s] or 0))[:top]:
        reasons = sorted(((c[6:], float(r[hdr.index(c)] or 0)) for c in cols), key=lambda x: -x[1])[:3]
        print(f"{float(r[i_s])/T*100:5.1f}% {r[i_a][-5:]} {r[i_src][:60]:60s} " + " ".join(f"{n}:{v/T*100:.1f}" for n, v in reasons if v))

if __name__ == "__main__" and "--stalls" in sys.argv:
    stall_table(sys.argv[1])
