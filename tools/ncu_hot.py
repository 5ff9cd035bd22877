"""Top stalled SASS instructions of an ncu report (source page), with context.
python tools/ncu_hot.py report.ncu-rep [N]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
tot = sum(int(d["Warp Stall Sampling (All Samples)"] or 0) for d in data)
print("total samples", tot, "instructions", len(data))
idx = sorted(range(len(data)), key=lambda i: -int(data[i]["Warp Stall Sampling (All Samples)"] or 0))
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
for i in idx[:N]:
    d = data[i]
    s = int(d["Warp Stall Sampling (All Samples)"] or 0)
    top = sorted(((int(d[h] or 0), h[6:]) for h in stalls), reverse=True)[:2]
    ctx = " | ".join(data[j]["Source"].strip()[:40] for j in range(max(0, i - 2), i))
    print(f"{100*s/tot:5.1f}% {d['Address'][-5:]} {d['Source'].strip()[:60]:60s} {top}  <- {ctx}")
