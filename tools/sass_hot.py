"""Per-instruction SASS hot spots from an ncu report (needs --import-source / -lineinfo)."""
import csv, subprocess, sys, io
rep = sys.argv[1]
topn = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
data = rows[2:]
ia, isrc = hdr.index("Address"), hdr.index("Source")
ist = hdr.index("Warp Stall Sampling (All Samples)")
iex = hdr.index("Instructions Executed")
ts = sum(float(r[ist] or 0) for r in data)
te = sum(float(r[iex] or 0) for r in data)
print(f"total stall samples {ts:.0f}, instructions {te:.3g}")
mode = sys.argv[3] if len(sys.argv) > 3 else "exec"
key = iex if mode == "exec" else ist
idx = sorted(range(len(data)), key=lambda i: -float(data[i][key] or 0))[:topn]
for i in sorted(idx):
    r = data[i]
    print(f"{i:5d} {100*float(r[iex] or 0)/te:5.2f}%i {100*float(r[ist] or 0)/ts:5.2f}%s  {r[isrc][:90]}")

if mode == "windows":
    pass
